# compute-sanitizer over the whole hot path (tools/sanitize_cases.py), one process per case so a
# failure is attributed: memcheck, racecheck (shared-memory hazards), synccheck (barrier misuse),
# initcheck (uninitialised global reads).  Logs: gpurun_out/san/<tool>_<size>_<case>.log; one
# summary line per run in gpurun_out/san/summary.txt.
mkdir -p gpurun_out/san
SIZES=${SAN_SIZES:-"tiny paper"}
TOOLS=${SAN_TOOLS:-"memcheck racecheck synccheck initcheck"}
CASES=${SAN_CASES:-"build spmv bj_scaled_persistent bj_scaled_graph bj_graph bj_persistent ssor_ai ilu0 none dist contacts"}
for sz in $SIZES; do
  for tool in $TOOLS; do
    for c in $CASES; do
      log=gpurun_out/san/${tool}_${sz}_${c}.log
      timeout 600 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
        python tools/sanitize_cases.py $sz $c > $log 2>&1
      rc=$?
      echo "$tool $sz $c rc=$rc $(grep -h 'SUMMARY' $log | tr '\n' ' ')" | tee -a gpurun_out/san/summary.txt
    done
  done
done
