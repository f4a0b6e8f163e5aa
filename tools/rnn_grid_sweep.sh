# c5 recurrences: per-step time vs CTA count (DUET_RNN_GRID; one-CTA kernels) -- with row-block step
# sync, fewer CTAs holding more tiles pipeline one tile's epilogue under the next tile's MMAs, so the
# SM-time (CTAs x time) a recurrence costs its co-running branches may drop
for sh in "lstm 4096 256 128 64" "lstm 4096 512 256 32" "gru 4096 512 256 32" "gru 4096 1024 256 16"; do
  python tools/rnn_time.py $sh
  for g in 32 48 64 74 96 128 148; do DUET_RNN_GRID=$g python tools/rnn_time.py $sh; done
done
