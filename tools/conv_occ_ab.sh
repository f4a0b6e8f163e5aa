# 64-channel im2col conv: CTAs per SM (DUET_CONV_OCC: 2 = default, 2 stages of 2 k-blocks; 5 = two CTAs
# with 1-k-block stages; 3 / 4 CTAs with 1-k-block stages)
for o in 2 3 4 5 2 3 4 5; do
  for sh in "4096 8 64 64 3 1 1" "64 56 64 64 3 1 1"; do
    echo -n "occ=$o $sh: "; DUET_CONV_OCC=$o DUET_CONV_HALO=0 CONV_ONE_GRAPH=1 python tools/conv_one.py $sh 10 2>&1 | tail -1
  done
done
echo -n "halo (c4 default) 64 56: "; CONV_ONE_GRAPH=1 python tools/conv_one.py 64 56 64 64 3 1 1 10 2>&1 | tail -1
