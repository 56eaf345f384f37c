for v in named; do
  for d in f32 f16; do for s in 0.2 0.95; do
  echo "$d $s"; CSWAP_GRAPHS=0 CSWAP_ZVC_PROF=1 CSWAP_LIB_VARIANT=$v timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s $s --dtype $d --reps 3 2>&1 | grep -E "zprof" | tail -1
  done; done
done
