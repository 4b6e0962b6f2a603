python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_fused_gather.py -q -x > gpurun_out/r03_pytest_f4.log 2>&1; echo "f4 rc=$?"; tail -30 gpurun_out/r03_pytest_f4.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/r03_pytest_gpu.log 2>&1; echo "all rc=$?"; tail -3 gpurun_out/r03_pytest_gpu.log
