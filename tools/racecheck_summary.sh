#!/bin/bash
# racecheck over tools/sanitize_run.py; the hazard report is summarised by (kind, source lines).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 compute-sanitizer --tool racecheck --racecheck-report all --print-limit 1000000 python tools/sanitize_run.py --ends ${ENDS:-300} ${CLASSES:+--classes $CLASSES} > /tmp/rc.log 2>&1
echo "racecheck rc=$?"
grep -E "parity|SUMMARY" /tmp/rc.log > gpurun_out/r02_racecheck_summary.txt
python - >> gpurun_out/r02_racecheck_summary.txt <<'PY'
import re, collections
c = collections.Counter()
kind = None
lines = []
for l in open("/tmp/rc.log"):
    m = re.search(r"(Error|Warning): (.*hazard)", l)
    if m:
        if kind: c[(kind, tuple(lines))] += 1
        kind, lines = m.group(1) + ": " + m.group(2), []
        continue
    m = re.search(r"(Read|Write|Atomic)\w* Thread.*in (\S+:\d+)", l)
    if m and kind: lines.append(m.group(1) + "@" + m.group(2))
if kind: c[(kind, tuple(lines))] += 1
for (k, ls), n in c.most_common(40):
    print(n, k, " | ".join(ls))
PY
cat gpurun_out/r02_racecheck_summary.txt | tail -45
