# h k-block order rotated per CTA (DUET_RNN_HROT=1 / 3, default 1) vs every CTA in order (0)
for m in 1 0 3 1 0 3; do
  for sh in "lstm 256 512 256 64" "gru 64 1024 256 64" "gru 4096 1024 256 16" "lstm 4096 512 256 32" "lstm 4096 256 128 64"; do
    DUET_RNN_HROT=$m python tools/rnn_time.py $sh | sed "s/^/hrot=$m /"
  done
done
