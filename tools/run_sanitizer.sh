# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize_run.py workloads (through gpurun)
mkdir -p gpurun_out
OUT=gpurun_out/sanitizer_${1:-run}.log
: > $OUT
for tool in memcheck racecheck synccheck; do
  for cfg in "C1 64 auto" "C2 1024 chain" "C2 1000 tile 1" "composite8 16 auto"; do
    echo "== $tool $cfg" >> $OUT
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py $cfg >> $OUT 2>&1
    echo "rc=$?" >> $OUT
  done
done
