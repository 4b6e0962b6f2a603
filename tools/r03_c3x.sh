python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_c3x.log; rm -f $L
for V in "T=0" "T=1" "T=2"; do
  echo "== $V" >> $L
  env POLYCONV_HK_$V POLYCONV_HK_VERBOSE=1 HK_DBGS="8" timeout 300 python tools/hk_trace.py 32 128 28 28 128 3 3 >> $L 2>&1
done
echo "== WSLOTS3 STREAM" >> $L
POLYCONV_HK_STREAM=1 POLYCONV_HK_VERBOSE=1 HK_DBGS="8" timeout 300 python tools/hk_trace.py 32 128 28 28 128 3 3 >> $L 2>&1
echo "== STREAM T1" >> $L
POLYCONV_HK_STREAM=1 POLYCONV_HK_T=1 POLYCONV_HK_VERBOSE=1 HK_DBGS="8" timeout 300 python tools/hk_trace.py 32 128 28 28 128 3 3 >> $L 2>&1
