#!/bin/bash
# task-granularity (KRCV_WIN_NBC) and rows-per-lane (KRCV_WIN_K) sweep on C2-C5
TAG=${1:-r01bc}; OUT=gpurun_out; mkdir -p $OUT
run() { timeout 300 python bench.py --config $1 --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_$2.json 2>/dev/null; }
for nbc in 20 30 40 60; do KRCV_WIN_NBC=$nbc run C2 C2_nbc$nbc; done
for K in 1 3; do KRCV_WIN_K=$K run C2 C2_K$K; done
for nbc in 6 13 26 52; do KRCV_WIN_NBC=$nbc run C3 C3_nbc$nbc; done
for nbc in 3 7 14 28; do KRCV_WIN_NBC=$nbc run C5 C5_nbc$nbc; done
for nbc in 1 2 4 8; do KRCV_WIN_NBC=$nbc run C4 C4_nbc$nbc; done
echo done
