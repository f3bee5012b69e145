#!/bin/bash
# ThreadSanitizer run of the loader / issuer host logic:
# libpask_testing.so rebuilt with -fsanitize=thread into _build/tsan/, then the
# fake-driver tests (tests/test_loader_fake.py: loader thread, work-stealing
# issuer, helper-thread encode, interleave, promote, destroy with queued loads)
# run against it with libtsan preloaded into the (uninstrumented) interpreter.
# Any TSAN report fails the run (halt_on_error=1, exitcode 66).
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
PKG=$ROOT/paper_conf_dac_huangdxz25_b200
OUT=$PKG/_build/tsan
mkdir -p "$OUT"
python -c "import sys; sys.path.insert(0, '$ROOT'); from paper_conf_dac_huangdxz25_b200 import build as b; b.build()"
FLAGS="-O1 -g -std=c++17 -fPIC -fsanitize=thread -fvisibility=hidden -I/usr/local/cuda/include -I$PKG/_build"
for f in pask plan driver fake_driver; do
  g++ $FLAGS -c "$PKG/csrc/runtime/$f.cpp" -o "$OUT/$f.o"
done
g++ -fsanitize=thread -shared -o "$OUT/libpask_testing.so" "$OUT"/pask.o "$OUT"/plan.o "$OUT"/driver.o \
    "$OUT"/fake_driver.o "$PKG/_build/fatbin.o" -ldl -lpthread \
    -Wl,--version-script="$PKG/csrc/runtime/exports.map"
cd "$ROOT"
TSAN_OPTIONS="halt_on_error=1 exitcode=66 report_signal_unsafe=0 second_deadlock_stack=1" \
PASK_TESTING_LIB="$OUT/libpask_testing.so" \
LD_PRELOAD=$(gcc -print-file-name=libtsan.so) \
python -m pytest tests/test_loader_fake.py -q -p no:cacheprovider "$@"
