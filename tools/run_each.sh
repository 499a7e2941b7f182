#!/bin/bash
# Run every test of the given files one by one under a hard timeout; one line each.
# usage: tools/run_each.sh SECONDS out.txt tests/file.py [...]
T=$1; OUT=$2; shift 2
: > "$OUT"
for f in "$@"; do
  for id in $(python -m pytest "$f" -m gpu --collect-only -q -p no:cacheprovider 2>/dev/null | grep "::"); do
    s=$(date +%s)
    timeout "$T" python -m pytest "$id" -m gpu -q -x -p no:cacheprovider > /tmp/one.log 2>&1
    rc=$?
    e=$(date +%s)
    echo "$id rc=$rc $((e - s))s" >> "$OUT"
    if [ $rc -ne 0 ]; then tail -25 /tmp/one.log >> "$OUT"; fi
  done
done
