# staged loader: GPU tests, then per-layer timing staged vs register loader
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || { tail -20 gpurun_out/r03_build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/r03_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r03_pytest_gpu.log
L=gpurun_out/r03_stg.log; rm -f $L
for SHAPE in "32 128 28 28 128 3 3" "256 64 56 56 64 3 3" "256 128 28 28 128 3 3" "64 256 56 56 256 3 3"; do
  for ST in "0 2" "1 2" "1 1"; do
    set -- $ST
    echo "== $SHAPE STAGED=$1 SBUFS=$2" >> $L
    POLYCONV_HK_STAGED=$1 POLYCONV_HK_SBUFS=$2 POLYCONV_HK_VERBOSE=1 HK_DBGS="8 9" timeout 200 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done
done
