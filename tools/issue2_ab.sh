# second x / h TMA issuer warp (DUET_RNN_ISSUE2=1, default) vs one (0) on the recurrences
for r in 1 2; do
  for m in 1 0; do
    for sh in "lstm 256 512 256 64" "gru 64 1024 256 64" "lstm 4096 256 128 64" "lstm 4096 512 256 32" \
              "gru 4096 512 256 32" "gru 4096 1024 256 16"; do
      DUET_RNN_ISSUE2=$m timeout 60 python tools/rnn_time.py $sh | sed "s/^/issue2=$m /"
    done
    DUET_RNN_ISSUE2=$m DUET_RNN_BN=128 timeout 60 python tools/rnn_time.py gru 64 1024 256 64 | sed "s/^/issue2=$m bn128 /"
    DUET_RNN_ISSUE2=$m DUET_RNN_PAIR=0 timeout 60 python tools/rnn_time.py lstm 4096 512 256 32 | sed "s/^/issue2=$m nopair /"
    DUET_RNN_ISSUE2=$m DUET_RNN_PAIR=0 timeout 60 python tools/rnn_time.py gru 4096 1024 256 16 | sed "s/^/issue2=$m nopair /"
  done
done
