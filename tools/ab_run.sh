#!/bin/bash
# Interleaved A/B timing of prof_apply cases: libraries alternate every round.
# usage: bash tools/ab_run.sh "<cases>" <rounds> <lib1.so> <lib2.so> ...
CASES=$1; ROUNDS=$2; shift 2
for r in $(seq $ROUNDS); do
  for lib in "$@"; do
    echo "== $(basename $lib) round $r"
    SVB200_LIB=$lib timeout 300 python tools/prof_apply.py 30 5 $CASES 2>&1 | awk '{print "   " $0}'
  done
done
