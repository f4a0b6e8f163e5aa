#!/bin/bash
# Round-2 same-box A/B experiments (GPU box; run from the repo root):  bash tools/ab_r2.sh <name>
# Each prints one line per run; the logs quoted in DESIGN.md are under profiles/r2_*.log.
cfg_line() {  # config, extra bench args...: p50 / serial / speed-up and the chosen slots
  local c=$1; shift
  timeout 500 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
    --tail-samples 200 "$@" | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['slot_of'], d['schedule']['profile_t_ns'])"
}
RNN_SHAPES=("lstm 256 512 256 64" "gru 64 1024 256 64" "lstm 4096 256 128 64" "lstm 4096 512 256 32" \
            "gru 4096 512 256 32" "gru 4096 1024 256 16")
case "$1" in
  msync)   # row-block step sync (1 = policy, 0 = grid barrier, 2 = always)   -> r2_msync_ab.log
    for m in 1 0 2; do for sh in "${RNN_SHAPES[@]}"; do DUET_RNN_MSYNC=$m python tools/rnn_time.py $sh | sed "s/^/msync=$m /"; done; done ;;
  ctarel)  # one counter release per CTA (1) vs per epilogue warp (0)          -> r2_ctarel_ab.log
    for m in 1 0 1 0; do for sh in "${RNN_SHAPES[@]:0:3}"; do DUET_RNN_CTAREL=$m python tools/rnn_time.py $sh | sed "s/^/ctarel=$m /"; done; done ;;
  hrot)    # rotated h k-block order (1) vs in order (0)                        -> r2_hrot_ab.log
    for m in 1 0 1 0; do for sh in "${RNN_SHAPES[@]}"; do DUET_RNN_HROT=$m python tools/rnn_time.py $sh | sed "s/^/hrot=$m /"; done; done ;;
  conv_occ)  # 64-channel convs: CTAs per SM (DUET_CONV_OCC 1/2/3/4)           -> r2_conv_occ.log
    for o in 2 3 4; do for sh in "4096 8 64 64 3 1 1" "64 56 64 64 3 1 1"; do
      echo -n "occ=$o $sh: "; DUET_CONV_OCC=$o CONV_ONE_GRAPH=1 python tools/conv_one.py $sh 10 2>&1 | tail -1; done; done ;;
  conv_occ128)  # 128-wide tiles: one (1) vs two (2) CTAs per SM                -> r2_conv_occ128.log
    for o in 1 2; do for sh in "64 28 128 128 3 1 1" "64 14 256 256 3 1 1" "64 7 512 512 3 1 1" "4096 4 128 128 3 1 1" \
                               "4096 2 256 256 3 1 1" "64 56 64 128 3 2 1" "4096 8 64 128 3 2 1"; do
      echo -n "occ128=$o $sh: "; DUET_CONV_OCC128=$o CONV_ONE_GRAPH=1 python tools/conv_one.py $sh 10 2>&1 | tail -1; done; done ;;
  conv_cfg)  # whole configs with the 128-wide conv choice auto (0) vs one CTA (1) -> r2_conv_cfg_ab.log
    for c in c4 c5; do for m in 0 1 0 1; do echo -n "$c occ128=$m: "; DUET_CONV_OCC128=$m cfg_line $c; done; done ;;
  measure_flush)  # measured Step 3 from a cold L2 (1) vs warm back-to-back (0) -> r2_measure_flush_ab.log
    for c in c5 c4 c2; do for m in 1 0 1 0; do echo -n "$c flush=$m: "; DUET_MEASURE_FLUSH=$m cfg_line $c; done; done ;;
  slots)   # c5 on 2 vs 3 stream slots
    for r in 1 2 3; do for n in 2 3; do echo -n "c5 slots=$n: "; cfg_line c5 --slots $n; done; done ;;
  pool)    # staged max pool (tools/pool_time.py; DUET_LIB=<older libduet.so> for the previous kernel)
    for sh in "64 112 112 64" "4096 16 16 64"; do python tools/pool_time.py $sh; done ;;
  embed)   # token-embedding gathers (tools/embed_time.py)                       -> r2_embed_ab.log
    for sh in "32 4096 256" "64 4096 128" "16 4096 256" "64 256 256" "64 64 256"; do python tools/embed_time.py $sh; done ;;
  refine)  # interleaved re-measurement of the 4 best candidates (4) vs Step 3's first figures (0)
    for r in 1 2 3; do for m in 4 0; do for c in c5 c4; do echo -n "$c refine=$m: "; DUET_MEASURE_REFINE=$m cfg_line $c; done; done; done ;;
  lstm_pair)  # LSTM on the CTA-pair recurrence (2, default) vs GRU only (1)     -> r2_lstm_pair_ab.log
    for m in 2 1 2 1; do for sh in "lstm 4096 512 256 32" "gru 4096 512 256 32"; do DUET_RNN_PAIR=$m python tools/rnn_time.py $sh | sed "s/^/pair=$m /"; done; done ;;
  *) echo "usage: bash tools/ab_r2.sh msync|ctarel|hrot|conv_occ|conv_occ128|conv_cfg|measure_flush|slots|pool|embed|refine|lstm_pair"; exit 1 ;;
esac
