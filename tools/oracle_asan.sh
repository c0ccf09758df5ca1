#!/bin/bash
# The oracle under AddressSanitizer + UBSan (SURVEY §5 "ASan on the oracle"): builds an instrumented
# copy of oracle/oracle.c and runs the CPU oracle pins (tests/test_oracle.py) against it.
set -e
cd "$(dirname "$0")/.."
gcc -O1 -g -fno-omit-frame-pointer -fsanitize=address,undefined -fopenmp -fPIC -shared -ffp-contract=off \
    -o /tmp/liboracle_asan.so oracle/oracle.c -lm
LD_PRELOAD="$(gcc -print-file-name=libasan.so):$(gcc -print-file-name=libubsan.so)" \
ASAN_OPTIONS=detect_leaks=0 UBSAN_OPTIONS=print_stacktrace=1:halt_on_error=1 ORACLE_LIB=/tmp/liboracle_asan.so \
    python -m pytest tests/test_oracle.py -q -p no:cacheprovider "$@"
