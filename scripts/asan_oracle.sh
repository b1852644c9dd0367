#!/bin/bash
# Build the C oracle with AddressSanitizer + UBSan and run a fuzz of solves through it
# (sanitizers on the oracle).  Prints "asan ok" and any sanitizer error.
set -e
cd "$(dirname "$0")/.."
gcc -O1 -g -std=c11 -ffp-contract=off -fopenmp -fsanitize=address,undefined -fno-omit-frame-pointer \
    -fPIC -shared -o /tmp/liboracle_asan.so oracle/madpipe_oracle.c -lm
cat > /tmp/asan_test.py <<'PY'
import sys
sys.path.insert(0, '.')
import oracle
oracle._LIB = '/tmp/liboracle_asan.so'
oracle.build = lambda force=False: '/tmp/liboracle_asan.so'
import numpy as np, chaingen
rng = np.random.default_rng(3)
for i in range(40):
    L = int(rng.integers(1, 12)); P = int(rng.integers(1, 5))
    ch = chaingen.tiny(rng, L)
    M = int((3*ch['W'].sum() + 3*ch['a'].sum())*rng.uniform(0.1, 0.9)) + 1
    oracle.solve(ch, P, M, float(rng.uniform(5, 50)), int(rng.choice([2, 4, 11])), int(rng.choice([3, 16])), 9,
                 v_range=int(rng.integers(0, 2)), n_threads=2)
    oracle.literal_solve(ch, P, M, 20.0, 4, 8, 11, K=4)
print("asan ok")
PY
LD_PRELOAD=$(gcc -print-file-name=libasan.so):$(gcc -print-file-name=libubsan.so) ASAN_OPTIONS=detect_leaks=0 \
    python /tmp/asan_test.py 2>&1 | grep -E "asan ok|ERROR|runtime error" || true
