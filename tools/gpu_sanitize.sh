# compute-sanitizer logs (memcheck, racecheck, synccheck, initcheck) of small runs
set -x
O=gpurun_out/sanitize; mkdir -p $O
for c in c1 c2 rl gs lean dump colony; do
  for t in memcheck racecheck synccheck; do
    SAN_CASE=$c timeout 900 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_run.py > $O/${c}_${t}.log 2>&1
    echo "exit $?" >> $O/${c}_${t}.log
  done
done
SAN_CASE=c1 timeout 900 compute-sanitizer --tool initcheck --print-limit 20 python tools/sanitize_run.py > $O/c1_initcheck.log 2>&1; echo "exit $?" >> $O/c1_initcheck.log
grep -H "ERROR SUMMARY\|RACECHECK SUMMARY\|parity\|^exit" $O/*.log
