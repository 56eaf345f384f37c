# recalibrate the selector's time models on the box with the current kernels, then the bench
# lines (VGG16 incl. extras / decision accuracy, BERT) with the new calibration
set -x
cp calib/b200.json gpurun_out/b200_calib_before.json
timeout 1800 python bench.py --calibrate --steps 3 --no-cpu > gpurun_out/calibrate.log 2>&1
cp calib/b200.json gpurun_out/b200_calib.json
timeout 900 python bench.py > gpurun_out/r_bench.json 2> gpurun_out/r_bench.err
timeout 900 python bench.py --workload bert --no-cpu > gpurun_out/r_bench_bert.json 2> gpurun_out/r_bench_bert.err
timeout 900 python bench.py --workload resnet50 --no-cpu > gpurun_out/r_bench_resnet.json 2> gpurun_out/r_bench_resnet.err
