# bench.py twice back to back (step-time spread across runs on one box) + the reference arm
mkdir -p gpurun_out
for i in 1 2; do timeout 900 python bench.py > gpurun_out/b2_$i.json 2> gpurun_out/b2_$i.err; done
timeout 600 python bench.py --impl reference > gpurun_out/b2_ref.json 2> gpurun_out/b2_ref.err
python -c "
import json
for f in ['gpurun_out/b2_1.json','gpurun_out/b2_2.json']:
    r=json.loads(open(f).read().strip().splitlines()[-1]); x=r['extras']
    print(f, r['value'], r['ms_per_step'], r['roofline']['frac'], r['roofline']['device_clock']['frac'], x['latency_ms'], x['link'], r['e2e']['value'])
print(open('gpurun_out/b2_ref.json').read().strip().splitlines()[-1][:400])"
