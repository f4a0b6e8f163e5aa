# ResNet conv layers as plain GEMMs (A materialised): one-CTA tiles vs CTA-pair tiles
for sh in "50176 128 1152" "12544 256 2304" "3136 512 4608" "65536 128 1152" "16384 256 2304" "200704 64 576"; do
  for bn in 64 128 256; do DUET_GEMM=1 DUET_GEMM_BN=$bn python tools/gemm_shape_time.py $sh; done
  for bn in 64 128 256; do DUET_GEMM_BN=$bn python tools/gemm_shape_time.py $sh; done
done
