# Loader fallback: a capped group kernel with local memory is rebuilt without the cap (NVRTC's
# cached results carry no ptxas log).  Register test 3x on the same box, then the GPU suite,
# smoke and the default bench.
set -x
for i in 1 2 3; do timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k test_registers_within_model_and_no_spills > gpurun_out/s4e_t$i.log 2>&1; done
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/s4e_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/s4e_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s4e_smoke.log 2>&1; echo "smoke rc $?" >> gpurun_out/s4e_smoke.log
timeout 900 python bench.py > gpurun_out/s4e_bench.json 2> gpurun_out/s4e_bench.err
