M=gpurun_out/s12; mkdir -p $M
timeout 1500 compute-sanitizer --tool initcheck --error-exitcode 9 --print-limit 4000 python tools/sanitize_run.py > $M/initcheck.log 2>&1; echo "initcheck rc=$?"; tail -3 $M/initcheck.log
grep -A6 "Uninitialized" $M/initcheck.log | grep "Device Frame" | sed 's/+0x[0-9a-f]*//' | sort | uniq -c | sort -rn | head -20
grep -A30 "Uninitialized" $M/initcheck.log | grep "Host Frame: granii::" | sed 's/\[0x.*//' | sort | uniq -c | sort -rn | head -20
