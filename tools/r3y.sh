python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 300 python tools/sanitize_cases.py
for t in memcheck synccheck racecheck; do timeout 1200 compute-sanitizer --tool $t python tools/sanitize_cases.py > gpurun_out/r3y_$t.log 2>&1; echo "$t rc $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|Race reported|hazard" gpurun_out/r3y_$t.log | sed 's/(.*//' | sort | uniq -c | head -8; done
