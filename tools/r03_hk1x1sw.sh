# mac_hankel tiling on the wide 1x1 layers it serves (NN x T x acc1)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r03_build.log 2>&1 || exit 1
L=gpurun_out/r03_hk1x1sw.log; rm -f $L
for SHAPE in "256 2048 7 7 512 1 1 1 0" "256 1024 14 14 512 1 1 1 0" "256 1024 14 14 256 1 1 1 0"; do
  echo "== $SHAPE default" >> $L; HK_KERNEL=tc_hankel HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
  for NN in 64 128 256; do for T in 1 2 4; do
    echo "== $SHAPE NN=$NN T=$T" >> $L; POLYCONV_HK_NN=$NN POLYCONV_HK_T=$T HK_KERNEL=tc_hankel HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
  done; done
  echo "== $SHAPE NN=256 T=1 acc0" >> $L; POLYCONV_HK_NN=256 POLYCONV_HK_T=1 POLYCONV_HK_ACC1=0 HK_KERNEL=tc_hankel HK_DBGS="0" timeout 60 python tools/hk_trace.py $SHAPE >> $L 2>&1
done
