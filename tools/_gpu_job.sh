i=0
for d in "" "-DMICCO_BARRIER_LATE=0" "-DMICCO_KEEP_SN=0" "-DMICCO_BARRIER_LATE=0 -DMICCO_KEEP_SN=0"; do
  i=$((i+1))
  MICCO_NVCC_DEFS="$d" python tools/build.py lib --force > /dev/null 2>&1 || echo BUILD FAIL
  python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_ab$i.log 2>&1
  python - <<PY
import json; d=json.loads(open("gpurun_out/bench_ab$i.log").read().strip().split("\n")[-1])
print("defs [$d]", round(d["value"]), d["roofline"]["achieved"], d["roofline"]["executed_frac"], d["breakdown_ms_per_step"])
PY
done
