# conv kernels A/B: halo vs im2col (DUET_CONV_HALO=0) at the ResNet shapes of c4 / c5
mkdir -p gpurun_out
for sh in "64 56 64 64 3 1 1" "64 28 128 128 3 1 1" "64 14 256 256 3 1 1" "4096 8 64 64 3 1 1"; do
  echo -n "halo   "; python tools/conv_one.py $sh 10
  echo -n "im2col "; DUET_CONV_HALO=0 python tools/conv_one.py $sh 10
done
