# im2col conv: W on its own issuing warp (DUET_CONV_ISS=2, default for one / two CTAs per SM) vs one producer (1)
for r in 1 2; do
  for m in 2 1; do
    for sh in "64 28 128 128 3 1 1" "64 14 256 256 3 1 1" "64 7 512 512 3 1 1" "4096 4 128 128 3 1 1" "4096 2 256 256 3 1 1" "64 56 64 128 3 2 1"; do
      echo -n "iss=$m $sh: "; DUET_CONV_ISS=$m CONV_ONE_GRAPH=1 timeout 120 python tools/conv_one.py $sh 10 2>&1 | tail -1
    done
  done
done
