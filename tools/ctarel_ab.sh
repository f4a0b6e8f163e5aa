# one-tile recurrence: one counter release per CTA (DUET_RNN_CTAREL=1) vs per epilogue warp (0),
# with the grid barrier and with row-block sync (DUET_RNN_MSYNC=2)
for r in 1 2; do
  for cfg in "0 1" "1 1" "0 2" "1 2"; do
    set -- $cfg
    for sh in "lstm 256 512 256 64" "gru 64 1024 256 64" "lstm 4096 256 128 64"; do
      DUET_RNN_CTAREL=$1 DUET_RNN_MSYNC=$2 python tools/rnn_time.py $sh | sed "s/^/ctarel=$1 msync=$2 /"
    done
  done
done
