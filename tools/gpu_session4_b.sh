# session 4: compute-sanitizer over small cases of every path on HEAD (adds the rank front and the
# two-level scatter + shared-memory bucket tables)
mkdir -p gpurun_out
O=gpurun_out/r1h_sanitizers.txt
echo "# round 1h: compute-sanitizer over tools/sanitize_cases.py (every path incl. rank front, two-level scatter, bucket tables)" > $O
for t in memcheck racecheck synccheck; do
  echo "== $t" >> $O
  timeout 900 compute-sanitizer --tool $t python tools/sanitize_cases.py >> $O 2>&1
  echo "rc=$?" >> $O
done
grep -E "^==|SUMMARY|rc=" $O
