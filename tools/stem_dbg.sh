# stem kernel component costs (DUET_STEM_DBG bits: 1 build, 2 MMA, 4 stores, 8 patch TMA skipped)
for d in 0 1 2 4 8 15; do
  echo -n "dbg=$d  "; DUET_STEM_DBG=$d python tools/node_times.py c4 2>&1 | grep cnn_stem
done
