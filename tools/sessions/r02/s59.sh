# compute-sanitizer over the final tree (entry-tile SDDMM and the new GAT reductions included)
M=gpurun_out/s59; mkdir -p $M
timeout 300 python tools/sanitize_run.py > $M/plain.log 2>&1; echo "plain rc=$?"; tail -2 $M/plain.log
for tool in memcheck racecheck initcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_run.py > $M/$tool.log 2>&1; echo "$tool rc=$?"; tail -4 $M/$tool.log
done
