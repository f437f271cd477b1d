# compute-sanitizer (memcheck / racecheck / synccheck) over tools/sanitize.py with
# kernel 4 forced, static-only and with the dynamic tail forced on at this size.
O=gpurun_out/san4
mkdir -p $O
for tool in memcheck racecheck synccheck; do
  CHECL_KERNEL=4 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_4.log 2>&1
  CHECL_KERNEL=4 CHECL_DYN_MIN_ROUNDS=0 CHECL_STATIC_PERMILLE=300 CHECL_DYN_BLOCK=2 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py > $O/san_${tool}_4dyn.log 2>&1
done
for f in $O/san_*.log; do echo "== $(basename $f)"; grep -E "sanitize ok|SUMMARY" $f; done > $O/sanitizer.txt
