python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_pphase.log; rm -f $L
for SHAPE in "256 512 14 14 512 3 3 2 1" "256 256 14 14 256 3 3 2 1" "64 128 14 14 128 3 3 2 1"; do
  for PL in 0 1 0 1; do echo "== $SHAPE PL=$PL" >> $L; POLYCONV_HK_PLANES=$PL POLYCONV_HK_VERBOSE=1 HK_DBGS="0" timeout 300 python tools/hk_trace.py $SHAPE >> $L 2>&1; done
done
timeout 600 python bench.py --workload resnet50 --no-cpu-baseline --no-cudnn > gpurun_out/r03_bench_resnet50.json 2>/dev/null; echo "r50 rc=$?"
