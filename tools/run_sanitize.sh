# compute-sanitizer over tools/sanitize.py; every tool run bounded by its own timeout
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  echo "== $tool"
  CSWAP_GRAPHS=0 timeout ${TOOL_TIMEOUT:-900} compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > gpurun_out/san_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/san_$tool.log
  tail -4 gpurun_out/san_$tool.log
done
