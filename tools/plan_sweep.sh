mkdir -p gpurun_out
for sh in "64 7 512 512 3 1 1" "64 14 256 256 3 1 1" "64 28 128 128 3 1 1" "4096 2 256 512 3 2 1" "4096 4 128 128 3 1 1" "64 14 256 512 3 2 1"; do
 for bn in 64 128 256; do for ks in 1 2 3 4; do
  echo -n "bn=$bn ks=$ks "; DUET_CONV_BN=$bn python tools/conv_one.py $sh 8
 done; done
done > gpurun_out/r2_plan_sweep.log 2>&1
ncu --set full --clock-control none -k regex:conv_tma -c 1 -o gpurun_out/r2_conv_l4c4 env DUET_CONV_PLAN=256,2 python tools/conv_one.py 64 7 512 512 3 1 1 1 > /dev/null 2>&1
ncu -i gpurun_out/r2_conv_l4c4.ncu-rep --page details --csv > gpurun_out/r2_conv_l4c4_details.csv 2>&1
ncu -i gpurun_out/r2_conv_l4c4.ncu-rep --page raw --csv > gpurun_out/r2_conv_l4c4_raw.csv 2>&1
