# Nondeterministic register count of the 35-kernel weather group under kf_exec_create: dump the
# generated source and ptxas log of four separate runs of the register test.
set -x
for i in 1 2 3 4; do
  mkdir -p gpurun_out/s4d_dump$i
  KF_DUMP_DIR=gpurun_out/s4d_dump$i timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k test_registers_within_model_and_no_spills > gpurun_out/s4d_t$i.log 2>&1
  rm -f gpurun_out/s4d_dump$i/*.cubin gpurun_out/s4d_dump$i/kf_g[1-9]*
done
