"""Aggregate an ncu SASS source page (CSV) by CUDA source line.

  ncu -i rep.ncu-rep --page source --csv --print-source sass --launch-skip S --launch-count 1 > k.csv
  nvdisasm -g -c locassm.sm_100a.cubin > all.sass        (cubin from cuobjdump -xelf all liblocassm.so)
  python tools/ncu_lines.py k.csv all.sass [top]

The line map comes from the locally built library (same source, same compiler); offsets are taken
relative to the kernel's first instruction.  Prints per source line: % of stall samples, % of
executed warp instructions, average active threads and the top stall reasons.
"""
import collections
import csv
import re
import sys


def line_map(sass_path, kernel):
    m, cur, inside, fn = {}, None, False, None
    for l in open(sass_path):
        if l.startswith(".text.") and l.rstrip().endswith(":"):
            inside = l.strip()[6:-1] == kernel
            continue
        if not inside:
            continue
        g = re.match(r'\s*//## File "(.*)", line (\d+)', l)
        if g:
            cur = (g.group(1).rsplit("/", 1)[-1], int(g.group(2)))
            continue
        g = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
        if g:
            m[int(g.group(1), 16)] = cur
    return m


def main():
    csv_path, sass_path = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
    rows = list(csv.reader(open(csv_path)))
    kname = rows[0][1]
    hdr = rows[1]
    data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr) and r[0].startswith("0x")]
    seen, uniq = set(), []
    for d in data:   # the CSV may list every instruction twice
        if d["Address"] in seen:
            continue
        seen.add(d["Address"])
        uniq.append(d)
    base = min(int(d["Address"], 16) for d in uniq)
    # mangled name: find the .text section whose instruction count matches
    sass = open(sass_path).read()
    names = re.findall(r"^\.text\.(\S+):$", sass, re.M)
    want = None
    short = re.sub(r"\(.*", "", kname.replace("void ", ""))
    tmpl = re.search(r"<\(int\)(\d+), \(bool\)(\d)(?:, \(int\)(\d+))?>", kname)
    tsmall = re.search(r"k_small<\(int\)(\d+)(?:, \(int\)(\d+))?>", kname)
    for n in names:
        if "k_smem" in short and tmpl:
            pre = "_ZN2la6k_smemILi%sELb%sE" % (tmpl.group(1), tmpl.group(2))
            if tmpl.group(3):
                pre += "Li%sE" % tmpl.group(3)
            if n.startswith(pre):
                want = n
        elif tsmall:
            pre = "_ZN2la7k_smallILi%sE" % tsmall.group(1)
            if tsmall.group(2):
                pre += "Li%sE" % tsmall.group(2)
            if n.startswith(pre):
                want = n
        elif short.split("::")[-1] in n:
            want = want or n
    lm = line_map(sass_path, want)

    def f(x):
        try:
            return float(x)
        except ValueError:
            return 0.0

    stall_cols = [c for c in hdr if c.startswith("stall_") and "Not Issued" not in c]
    agg = collections.defaultdict(lambda: collections.Counter())
    for d in uniq:
        key = lm.get(int(d["Address"], 16) - base, ("?", 0))
        a = agg[key]
        a["samples"] += f(d["Warp Stall Sampling (All Samples)"])
        a["inst"] += f(d["Instructions Executed"])
        a["tinst"] += f(d["Thread Instructions Executed"])
        for c in stall_cols:
            a[c] += f(d[c])
    ts = sum(a["samples"] for a in agg.values()) or 1
    ti = sum(a["inst"] for a in agg.values()) or 1
    print(f"kernel {want}: {len(uniq)} SASS instructions, {ti:.3g} warp instructions executed")
    for key, a in sorted(agg.items(), key=lambda kv: -kv[1]["samples"])[:top]:
        st = sorted(((a[c], c[6:]) for c in stall_cols), reverse=True)[:3]
        thr = a["tinst"] / a["inst"] if a["inst"] else 0
        print(f"{key[0]}:{key[1]:<5} samp {100 * a['samples'] / ts:5.1f}%  inst {100 * a['inst'] / ti:5.1f}%  "
              f"thr {thr:4.1f}  " + " ".join(f"{n}={100 * v / max(a['samples'], 1):.0f}%" for v, n in st))


if __name__ == "__main__":
    main()
