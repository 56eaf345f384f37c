#!/bin/bash
# One gpurun batch for the NEXT rows' measurements (outputs under gpurun_out/, copied to profiles/)
set -x
timeout 900 python bench.py --calibrate --steps 3 --no-cpu > gpurun_out/calibrate.log 2>&1
cp calib/b200.json gpurun_out/b200_calib.json
timeout 600 python tools/launch_tune.py --out gpurun_out/launch_tune_r01.json > gpurun_out/launch_tune.log 2>&1
timeout 900 python tools/time_models.py --collect 60 --out gpurun_out/time_model_samples_r01.json > gpurun_out/time_models_collect.log 2>&1
timeout 900 python tools/drift.py > gpurun_out/drift_r01.jsonl 2>gpurun_out/drift.err
timeout 600 python bench.py --workload resnet50 --no-cpu > gpurun_out/bench_resnet50.log 2>&1
timeout 600 python bench.py --workload bert --no-cpu > gpurun_out/bench_bert.log 2>&1
for cfg in 0 1 2 3; do for m in 24 96 1024; do CSWAP_ZVC_CFG=$cfg python tools/codec_bench.py --codecs zvc --mib $m --s 0.5 2>&1 | tail -1 | sed "s/^/cfg$cfg /"; done; done > gpurun_out/zvc_cfg_sweep.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"zvc_(compress|expand|count)" -s 6 -c 6 -o gpurun_out/zvc_f32_micro -f python tools/codec_bench.py --codecs zvc --dtype f32 --s 0.5 --ncu > /dev/null 2>&1
timeout 900 python tools/train_step.py --model resnet50 > gpurun_out/train_resnet50.log 2>&1
