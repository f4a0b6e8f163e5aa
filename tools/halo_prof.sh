mkdir -p gpurun_out
bash tools/halo_ab.sh > gpurun_out/r2_halo_ab.log 2>&1
for sh in "64 56 64 64 3 1 1:l1c4" "4096 8 64 64 3 1 1:l1c5" "64 14 256 256 3 1 1:l3c4"; do
  args=${sh%%:*}; tag=${sh##*:}
  ncu --set full --clock-control none -k regex:conv_halo -c 1 -o gpurun_out/r2_halo_$tag python tools/conv_one.py $args 1 > /dev/null 2>&1
  ncu -i gpurun_out/r2_halo_$tag.ncu-rep --page raw --csv > gpurun_out/r2_halo_${tag}_raw.csv 2>&1
done
