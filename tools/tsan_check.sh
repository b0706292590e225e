#!/bin/bash
# Host-side ThreadSanitizer run (SURVEY.md §5 "host TSAN build"): builds a copy of libmicco.so
# whose host code is compiled with -fsanitize=thread (device code unchanged), swaps it into a
# scratch copy of the repo, and runs the GPU tests that exercise the executor's host threads
# (streamed planning thread + replay, per-GPU tables, evictions and peer copies) under it.
# Usage (on the GPU box): bash tools/tsan_check.sh [pytest -k expression]
set -u
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=${TSAN_OUT:-$ROOT/gpurun_out/tsan}
K=${1:-"streamed_planning or per_gpu_scalar_tables or c5_mixed or cross_run or keep_inputs or gpu_count_change or canonical"}
W=/tmp/micco_tsan
rm -rf "$W" && mkdir -p "$W/obj" "$OUT"
mkdir -p "$W/repo" && tar -C "$ROOT" --exclude=./build --exclude=./gpurun_out --exclude=./profiles -cf - . | tar -C "$W/repo" -xf -
NVCC=/usr/local/cuda/bin/nvcc
ARCH="-gencode arch=compute_100a,code=sm_100a"
SRC=$ROOT/paper_conf_ipps_wangr0e22_b200/csrc
INC="-I $ROOT/include -I $ROOT -I $SRC"
objs=()
for s in "$SRC"/*.cu "$SRC"/*.cpp; do
  o="$W/obj/$(basename "$s").o"
  $NVCC $ARCH -std=c++17 -O1 -g -Xcompiler -fPIC,-fsanitize=thread,-fno-omit-frame-pointer $INC -x cu -c "$s" -o "$o" &
  objs+=("$o")
done
wait
for o in "${objs[@]}"; do [ -f "$o" ] || { echo "compile failed: $o"; exit 1; }; done
$NVCC $ARCH -shared -cudart shared -Xcompiler -fsanitize=thread -o "$W/repo/paper_conf_ipps_wangr0e22_b200/libmicco.so" \
  "${objs[@]}" -lpthread -ldl -ltsan || exit 1
cd "$W/repo"
# harness check: a deliberately racy instrumented library must produce a report here
cat > "$W/racy.c" <<'EOC'
#include <pthread.h>
static int counter;
static void *bump(void *p) { for (int i = 0; i < 100000; ++i) counter++; return p; }
int racy(void) { pthread_t a, b; pthread_create(&a, 0, bump, 0); pthread_create(&b, 0, bump, 0);
                 pthread_join(a, 0); pthread_join(b, 0); return counter; }
EOC
gcc -shared -fPIC -g -fsanitize=thread -o "$W/libracy.so" "$W/racy.c"
export TSAN_OPTIONS="report_signal_unsafe=0 second_deadlock_stack=1 log_path=$OUT/harness halt_on_error=0"
LD_PRELOAD=$(gcc -print-file-name=libtsan.so) setarch "$(uname -m)" -R \
  python -c "import ctypes; ctypes.CDLL('$W/libracy.so').racy()"
grep -l "WARNING: ThreadSanitizer: data race" "$OUT"/harness.* 2>/dev/null | wc -l > "$OUT/harness_reports.txt"
export TSAN_OPTIONS="report_signal_unsafe=0 second_deadlock_stack=1 log_path=$OUT/tsan halt_on_error=0 ignore_noninstrumented_modules=1"
LD_PRELOAD=$(gcc -print-file-name=libtsan.so) setarch "$(uname -m)" -R \
  python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "$K" > "$OUT/pytest.txt" 2>&1
echo "pytest rc=$?" >> "$OUT/pytest.txt"
ls "$OUT"
grep -l "WARNING: ThreadSanitizer" "$OUT"/tsan.* 2>/dev/null | wc -l > "$OUT/n_reports.txt"
grep -h "WARNING: ThreadSanitizer\|#0 \|#1 " "$OUT"/tsan.* 2>/dev/null | head -200 > "$OUT/summary.txt"
tail -3 "$OUT/pytest.txt"
