#!/bin/bash
# GPU-box tasks (run through gpurun from the repo root): bash tools/gpu_tasks.sh TASK [TASK ...]
# Every task writes under gpurun_out/ (copied back by gpurun) and bounds each command with its own
# timeout.  Summaries worth keeping are copied into profiles/ (named per round) by hand.
#
#   tests      pytest -m gpu + __graft_entry__.smoke()
#   bench      bench.py (VGG16 set, incl. extras) + BERT / ResNet-50 sets + the reference arm
#   zvc        ZVC compress / decompress table: 1 GiB f32 / f16 / bf16 x s in {.2,.5,.8,.95}, and
#              f32 / f16 at 16 / 24 / 96 / 256 MiB (codec_bench.py; L2 flushed; clocks recorded)
#   sweep      BASELINE configs[1]: sizes x sparsities x 4 codecs, clustered, fp16 / bf16 (+ sweep_kinds)
#   sweep_kinds  clustered (L0 = 32), channel-dead, all-zero, dense at 64 MiB (appended to sweep.jsonl)
#   profiles   ncu launch list of the bench command + ncu --set full summaries of the bench step's
#              compress / decode launches and of the 1 GiB micro kernels (SASS mix, per-line)
#   sanitize   compute-sanitizer memcheck / racecheck / synccheck / initcheck on tools/sanitize.py
#   calibrate  re-fit calib/b200.json on the box (bench.py --calibrate)
#   next       NEXT-row measurements: launch_tune, time models, drift, training steps
#   pipeline   swap pipeline timeline / granularity probe (tools/pipeline_probe.py)
#   probes     event cost during copies (event_probe, event_gap_probe), D2H rates by allocation,
#              SM-driven vs copy-engine copies, host time of small codec calls, link ramp on a box
#   cpuplan    oracle CPU timing plan (bench.py --cpu-plan)
mkdir -p gpurun_out
R=/tmp/ncu_reps; mkdir -p $R
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_throttle_reasons.active --format=csv
for task in "$@"; do
  echo "== task $task"
  case $task in
  tests)
    timeout 1500 python -m pytest tests -q -m gpu -x -p no:cacheprovider > gpurun_out/t_pytest.log 2>&1; tail -3 gpurun_out/t_pytest.log
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/t_smoke.log 2>&1; echo "smoke rc=$?" | tee -a gpurun_out/t_smoke.log ;;
  bench)
    timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/b_bench.json 2> gpurun_out/b_bench.err
    timeout 900 python bench.py --workload bert --no-cpu > gpurun_out/b_bench_bert.json 2> gpurun_out/b_bench_bert.err
    timeout 900 python bench.py --workload resnet50 --no-cpu > gpurun_out/b_bench_resnet50.json 2> gpurun_out/b_bench_resnet50.err
    timeout 900 python bench.py --workload resnet50_f16 --no-cpu > gpurun_out/b_bench_resnet50_f16.json 2> gpurun_out/b_bench_resnet50_f16.err
    timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/b_reference.json 2> gpurun_out/b_reference.err ;;
  zvc)
    out=gpurun_out/z_zvc.jsonl; : > $out
    for d in f32 f16 bf16; do timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.2,0.5,0.8,0.95 --dtype $d --check >> $out 2>/dev/null; done
    for d in f32 f16; do for m in 16 24 96 256; do timeout 300 python tools/codec_bench.py --codecs zvc --mib $m --s 0.5,0.8,0.95 --dtype $d --check >> $out 2>/dev/null; done; done
    python tools/sweep_table.py $out > gpurun_out/z_zvc.md 2>&1; cat gpurun_out/z_zvc.md ;;
  sweep)
    rm -f gpurun_out/sweep.jsonl
    for mib in 0.0625 0.25 1 4 16 64 256 1024; do for c in zvc rle csr lz4; do
      reps=10; [ "$c" = lz4 ] && [ "$mib" = 1024 ] && reps=3
      timeout 600 python tools/codec_bench.py --codecs $c --mib $mib --s 0.0,0.05,0.1,0.2,0.3,0.4,0.5,0.6,0.7,0.8,0.9,0.95 --reps $reps --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
    done; done
    for c in zvc rle csr lz4; do timeout 600 python tools/codec_bench.py --codecs $c --mib 64 --s 0.5,0.8,0.95,0.99 --kind clustered --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err; done
    for d in f16 bf16; do timeout 600 python tools/codec_bench.py --codecs zvc,rle,csr,lz4 --mib 64 --s 0.2,0.5,0.8 --dtype $d --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err; done
    bash tools/gpu_tasks.sh sweep_kinds
    python tools/sweep_table.py gpurun_out/sweep.jsonl > gpurun_out/sweep.md 2>&1; wc -l gpurun_out/sweep.jsonl ;;
  sweep_kinds)  # the other zero structures of SURVEY §8(d) at 64 MiB, appended to sweep.jsonl
    for c in zvc rle csr lz4; do
      for kind in clustered32 dead; do timeout 600 python tools/codec_bench.py --codecs $c --mib 64 --s 0.5,0.8,0.95,0.99 --kind $kind --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err; done
      for kind in zero dense; do timeout 600 python tools/codec_bench.py --codecs $c --mib 64 --s 0.0 --kind $kind --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err; done
    done ;;
  profiles)
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/p_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/p_launches.log 2>&1
    python tools/launch_summary.py gpurun_out/p_launches.csv "python bench.py --steps 2 --warmup 3 --no-extras --no-cpu (under ncu: warm-up + timed steps of the VGG16 b64 set, then the isolated replay of the 12 tensors x 4)" > gpurun_out/p_launches.txt
    timeout 1200 ncu --set full --clock-control none -k regex:zvc_compress -s 37 -c 12 -o $R/bench_step -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu1.log 2>&1
    timeout 1200 ncu --set full --clock-control none -k regex:"zvc_(count|scan|expand)" -s 369 -c 30 -o $R/bench_dec -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu2.log 2>&1
    for d in f32 f16; do
      timeout 600 ncu --set full --import-source on --clock-control none -k regex:"zvc_(compress_persistent|expand)" -s 2 -c 2 -o $R/micro_$d -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype $d --ncu > gpurun_out/p_ncu_micro_$d.log 2>&1
      python tools/ncu_sass_mix.py $R/micro_$d.ncu-rep zvc_compress 25 > gpurun_out/p_sassmix_compress_$d.txt 2>&1
      python tools/ncu_lines.py $R/micro_$d.ncu-rep zvc_compress 40 > gpurun_out/p_lines_compress_$d.txt 2>&1
    done
    python tools/ncu_summary.py gpurun_out/p_ncu.json bench_step=$R/bench_step.ncu-rep bench_step_dec=$R/bench_dec.ncu-rep micro_1GiB_f32_s05=$R/micro_f32.ncu-rep micro_1GiB_f16_s05=$R/micro_f16.ncu-rep > /dev/null ;;
  sanitize)
    for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
      CSWAP_GRAPHS=0 timeout ${TOOL_TIMEOUT:-900} compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/san_$tool.log 2>&1
      echo "rc=$?" >> gpurun_out/san_$tool.log; echo "-- $tool"; tail -4 gpurun_out/san_$tool.log
    done ;;
  calibrate)
    cp calib/b200.json gpurun_out/b200_calib_before.json
    timeout 1800 python bench.py --calibrate --steps 3 --no-cpu > gpurun_out/calibrate.log 2>&1
    cp calib/b200.json gpurun_out/b200_calib.json ;;
  next)
    timeout 600 python tools/launch_tune.py --out gpurun_out/launch_tune.json > gpurun_out/launch_tune.log 2>&1
    timeout 900 python tools/time_models.py --collect 60 --out gpurun_out/time_model_samples.json > gpurun_out/time_models_collect.log 2>&1
    timeout 900 python tools/drift.py > gpurun_out/drift.jsonl 2> gpurun_out/drift.err
    timeout 900 python tools/train_step.py --model vgg16 > gpurun_out/train_vgg16.log 2>&1
    timeout 900 python tools/train_step.py --model resnet50 > gpurun_out/train_resnet50.log 2>&1 ;;
  pipeline)
    timeout 900 python tools/pipeline_probe.py > gpurun_out/pipeline_probe.jsonl 2> gpurun_out/pipeline_probe.err ;;
  probes)
    nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/evp tools/event_probe.cu && timeout 300 /tmp/evp > gpurun_out/event_probe.jsonl 2>&1
    nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/d2hp tools/d2h_probe.cu && timeout 300 /tmp/d2hp > gpurun_out/d2h_probe.jsonl 2>&1
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC tools/zc_probe.cu -o tools/zc_probe.so && timeout 300 python tools/zc_probe.py > gpurun_out/zc_probe.txt 2>&1
    nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/egp tools/event_gap_probe.cu && timeout 300 /tmp/egp > gpurun_out/event_gap_probe.txt 2>&1
    timeout 300 python tools/host_overhead_probe.py > gpurun_out/host_overhead.jsonl 2>&1
    timeout 120 python tools/fresh_box_probe.py > gpurun_out/fresh_box_probe.jsonl 2>&1
    nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/dip tools/d2h_interference_probe.cu && timeout 300 /tmp/dip > gpurun_out/d2h_interference.jsonl 2>&1 ;;
  cpuplan)
    timeout 1800 python bench.py --cpu-plan gpurun_out/cpu_plan.json > gpurun_out/cpu_plan.log 2>&1 ;;
  *) echo "unknown task $task" ;;
  esac
done
du -sh gpurun_out
