# compute-sanitizer (memcheck / racecheck / synccheck) over tools/sanitize.py with
# the graph launches (default), default kernel choice and kernel 3 / 4 forced.
O=gpurun_out/sang
mkdir -p $O
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_default.log 2>&1
  CHECL_KERNEL=3 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_3.log 2>&1
  CHECL_KERNEL=4 CHECL_DYN_MIN_ROUNDS=0 CHECL_STATIC_PERMILLE=300 CHECL_DYN_BLOCK=2 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_4dyn.log 2>&1
done
for f in $O/san_*.log; do echo "== $(basename $f)"; grep -E "sanitize ok|SUMMARY" $f; done > $O/sanitizer.txt
cat $O/sanitizer.txt
