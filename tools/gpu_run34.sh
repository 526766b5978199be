# A/B of the 64-column bf16 store boxes (prof build, env switch)
export PCNN_LIB=$PWD/build/prof/libpcnn_prof.so
for wide in 0 1; do
  if [ $wide = 0 ]; then export PCNN_NO_WIDE_STORE=1; else unset PCNN_NO_WIDE_STORE; fi
  echo "== no_wide=$((1-wide))"
  timeout -s KILL 300 python tools/ab_flags.py 256 0 2>&1 | tr -d '\n ' ; echo
  timeout -s KILL 300 python tools/ab_flags.py 64 0 2>&1 | tr -d '\n ' ; echo
  timeout -s KILL 300 python tools/rank_layers.py 2>&1 | tr -d '\n '; echo
done
