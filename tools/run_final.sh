# final-tree check: GPU tests, smoke, bench line, ZVC table
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu -x 2>&1 | tail -2
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/f_bench.json 2> gpurun_out/f_bench.err
python -c "
import json
r=json.loads(open('gpurun_out/f_bench.json').read().strip().splitlines()[-1]); x=r['extras']
print(r['value'], r['ms_per_step'], r['roofline']['frac'], r['roofline']['device_clock']['frac'], r['roofline']['isolated'], x['latency_ms'], x['link'], r['e2e']['value'], r['clocks'])"
bash tools/run_zvc_table.sh 2>&1 | tail -14
