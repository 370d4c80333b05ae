"""Per-launch DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of every kernel in an
ncu --set full report, merged into profiles/ncu_traffic.json (bench.py's roofline.traffic).

  python tools/ncu_traffic.py gpurun_out/prof.ncu-rep [profiles/ncu_traffic.json]
"""
import csv, io, json, os, subprocess, sys


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ix = {h: i for i, h in enumerate(hdr)}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    d = json.load(open(out)) if os.path.exists(out) else {}
    for r in data:
        tot = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            tot += float(r[ix[m]].replace(",", "")) * scale.get(units[ix[m]], 1)
        d[r[ix["Kernel Name"]]] = tot
        print(r[ix["Kernel Name"]], f"{tot / 1e9:.3f} GB")
    json.dump(d, open(out, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "profiles/ncu_traffic.json")
