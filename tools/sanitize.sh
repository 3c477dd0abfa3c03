# compute-sanitizer memcheck / synccheck / racecheck over tools/sanitize_cases.py, only the
# library's kernels (mstk::); logs -> gpurun_out/sanitize_<tool>.log (racecheck: the summary and
# the unique hazard locations; the full per-hazard listing can be hundreds of MB)
for tool in ${TOOLS:-memcheck synccheck racecheck}; do
  extra="--print-limit 100"
  [ "$tool" = "racecheck" ] && extra="--racecheck-report all --print-limit 100000"
  timeout ${TMO:-1500} compute-sanitizer --tool $tool $extra --kernel-name kns=mstk --target-processes all \
      --log-file /tmp/san_$tool.log python tools/sanitize_cases.py > gpurun_out/sanitize_$tool.out 2>&1
  echo "$tool rc=$?"
  if [ "$tool" = "racecheck" ]; then
    { grep -E "RACECHECK SUMMARY|ERROR SUMMARY" /tmp/san_$tool.log;
      echo "unique hazard locations (count, kernel, line):";
      grep -oE "at mstk::[a-zA-Z0-9_]+[^ ]* .*in [a-zA-Z0-9_.]+:[0-9]+" /tmp/san_$tool.log | \
        sed -E 's/\(.*\)\+0x[0-9a-f]+//' | sort | uniq -c | sort -rn | head -40; } > gpurun_out/sanitize_$tool.log
    head -c 4000000 /tmp/san_$tool.log | gzip > gpurun_out/sanitize_${tool}_head.log.gz
  else
    cp /tmp/san_$tool.log gpurun_out/sanitize_$tool.log
  fi
  tail -3 gpurun_out/sanitize_$tool.log; tail -2 gpurun_out/sanitize_$tool.out
done
