# 128-512-channel layers: 128-wide tiles (one CTA per SM, default) vs 64-wide tiles on three CTAs per SM
for bn in 128 64 128 64; do
  for sh in "64 28 128 128 3 1 1" "64 14 256 256 3 1 1" "64 7 512 512 3 1 1" "4096 4 128 128 3 1 1" "4096 2 256 256 3 1 1" "64 56 64 128 3 2 1"; do
    echo -n "bn=$bn $sh: "; DUET_CONV_BN=$bn CONV_ONE_GRAPH=1 python tools/conv_one.py $sh 10 2>&1 | tail -1
  done
done
