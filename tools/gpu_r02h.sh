python -c "import __graft_entry__ as g; g.build()"
rm -rf gpurun_out/san; mkdir -p gpurun_out/san
SAN_SIZES=tiny bash tools/gpu_sanitize.sh > /dev/null 2>&1
SAN_SIZES=paper SAN_TOOLS="memcheck racecheck synccheck" SAN_CASES="build spmv bj_scaled_persistent ssor_ai bj_persistent dist contacts" bash tools/gpu_sanitize.sh > /dev/null 2>&1
SAN_SIZES=paper SAN_TOOLS="initcheck" SAN_CASES="bj_scaled_persistent dist" bash tools/gpu_sanitize.sh > /dev/null 2>&1
cat gpurun_out/san/summary.txt
