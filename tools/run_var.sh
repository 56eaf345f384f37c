# bench step-time variance: old vs new calibration (no extras)
for i in 1 2; do
for c in old new; do
  if [ $c = new ]; then cp calib/b200_new.json calib/b200.json; else git_old=1; cp calib/b200_old.json calib/b200.json; fi
  timeout 600 python bench.py --no-cpu 2>/dev/null | python -c "
import sys,json
b=json.loads(sys.stdin.read().strip().splitlines()[-1]); l=b['extras']['latency_ms']
print('$c', b['ms_per_step'], 'auto', round(l['auto'],2), 'sc', round(l['sc_always_zvc'],2), 'none', round(l['vdnn_none'],2), b['config']['codecs_chosen'][:3])"
done; done
