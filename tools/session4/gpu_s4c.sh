# Reverted fill kernel (the row/column rewrite was slower: 10 vs 8 us per buffer).  Determinism
# check of test_registers_within_model_and_no_spills (failed once with local_bytes 8 on a reused
# box), then the whole GPU suite without -x.
set -x
mkdir -p gpurun_out/s4c_dump1 gpurun_out/s4c_dump2
KF_DUMP_DIR=gpurun_out/s4c_dump1 timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k test_registers_within_model_and_no_spills > gpurun_out/s4c_t1.log 2>&1
KF_DUMP_DIR=gpurun_out/s4c_dump2 timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k test_registers_within_model_and_no_spills > gpurun_out/s4c_t2.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/s4c_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/s4c_pytest_gpu.log
rm -f gpurun_out/s4c_dump*/*.cu
