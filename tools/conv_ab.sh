# 128-wide im2col conv: one CTA per SM with 2-k-block stages vs two CTAs with 1-k-block stages
for sh in "64 28 128 128 3 1 1" "64 14 256 256 3 1 1" "64 7 512 512 3 1 1" "4096 4 128 128 3 1 1" "4096 2 256 256 3 1 1" "64 56 64 128 3 2 1"; do
  for k in 0 1; do echo -n "k1=$k "; DUET_CONV_K1=$k python tools/conv_one.py $sh 10; done
done
