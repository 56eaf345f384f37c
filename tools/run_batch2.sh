set -x
timeout 900 python bench.py --calibrate --steps 3 --no-cpu > gpurun_out/calibrate.log 2>&1
cp calib/b200.json gpurun_out/b200_calib.json
timeout 600 python bench.py --workload bert --no-cpu > gpurun_out/bench_bert.log 2>&1
timeout 600 python tools/drift_diag.py 0.65 > gpurun_out/drift_diag_065.log 2>&1
timeout 900 python tools/drift.py > gpurun_out/drift_r01.jsonl 2>gpurun_out/drift.err
timeout 900 python tools/time_models.py --collect 60 --out gpurun_out/time_model_samples_r01.json > gpurun_out/time_models_collect.log 2>&1
