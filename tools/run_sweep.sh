# BASELINE.json configs[1]: sparsity sweep x sizes, all four codecs, compress / decompress GB/s
# (tools/codec_bench.py, L2 flushed between reps, round trip checked) -> gpurun_out/sweep.jsonl;
# plus ncu --set full summaries of every RLE / CSR / LZ4 kernel at 256 MiB s = 0.5.
set -x
rm -f gpurun_out/sweep.jsonl
for mib in 0.0625 1 16 256 1024; do
  for c in zvc rle csr lz4; do
    reps=10; [ "$c" = lz4 ] && [ "$mib" = 1024 ] && reps=3
    timeout 600 python tools/codec_bench.py --codecs $c --mib $mib --s 0.0,0.2,0.5,0.8,0.95 --reps $reps --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
  done
done
for kind in clustered; do for c in zvc rle csr lz4; do
  timeout 600 python tools/codec_bench.py --codecs $c --mib 256 --s 0.5,0.8,0.95 --kind $kind --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done; done
for d in f16 bf16; do timeout 600 python tools/codec_bench.py --codecs zvc,rle,csr,lz4 --mib 256 --s 0.2,0.5,0.8 --dtype $d --check >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err; done
R=/tmp/ncu_reps; mkdir -p $R
for c in rle csr lz4; do
  timeout 900 ncu --set full --clock-control none -k regex:"${c}_|prep_kernel|finalize_kernel" -o $R/codec_$c -f python tools/codec_bench.py --codecs $c --mib 256 --s 0.5 --ncu > gpurun_out/ncu_codec_$c.log 2>&1
done
python tools/ncu_summary.py gpurun_out/ncu_codecs.json rle_256MiB_s05=$R/codec_rle.ncu-rep csr_256MiB_s05=$R/codec_csr.ncu-rep lz4_256MiB_s05=$R/codec_lz4.ncu-rep > /dev/null
wc -l gpurun_out/sweep.jsonl; du -sh gpurun_out
