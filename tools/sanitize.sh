# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_cases.py, only the
# library's kernels (mstk::); logs -> gpurun_out/sanitize_<tool>.log
for tool in ${TOOLS:-memcheck synccheck racecheck}; do
  extra=""
  [ "$tool" = "racecheck" ] && extra="--racecheck-report hazard"
  timeout ${TMO:-1500} compute-sanitizer --tool $tool $extra --kernel-name regex:mstk --target-processes all \
      --print-limit 50 --log-file gpurun_out/sanitize_$tool.log \
      python tools/sanitize_cases.py > gpurun_out/sanitize_$tool.out 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize_$tool.log; tail -2 gpurun_out/sanitize_$tool.out
done
