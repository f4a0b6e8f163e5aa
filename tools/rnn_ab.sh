# GRU timing A/B: current libduet vs tools/ab/libduet_r2base.so (DUET_LIB), c4 / c5 GRU shapes
for lib in paper_conf_ipps_zhanghl21_b200/libduet.so tools/ab/libduet_r2base.so; do
  echo "== $lib"
  for sh in "gru 4096 1024 256 16" "gru 4096 512 256 32" "gru 64 1024 256 64" "lstm 4096 512 256 32"; do
    echo -n "$sh: "; DUET_LIB=$lib python tools/rnn_time.py $sh
  done
done
