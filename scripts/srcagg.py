"""Aggregate `ncu --page source --csv --print-source cuda,sass` by CUDA source line from its SASS rows
(robust to source text that breaks the CSV quoting).  usage: srcagg.py CSV SRCFILE [N]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
src = open(sys.argv[2]).read().split("\n")
n = int(sys.argv[3]) if len(sys.argv) > 3 else 40
cur = None
samp = collections.Counter(); inst = collections.Counter(); thr = collections.Counter()
for r in rows[3:]:
    if r and r[0]:
        try: cur = int(r[0])
        except ValueError: pass
        continue
    if len(r) > 8 and r[2].startswith("0x"):
        try:
            samp[cur] += int(r[4] or 0); inst[cur] += int(r[7] or 0); thr[cur] += int(r[8] or 0)
        except ValueError: pass
ts = sum(samp.values()) or 1; ti = sum(inst.values()) or 1
print(f"samples {ts}  warp-inst {ti:.3e}  threads/inst {sum(thr.values())/ti:.1f}")
for ln, s in samp.most_common(n):
    t = thr[ln] / inst[ln] if inst[ln] else 0
    print(f"{100*s/ts:5.1f}% inst {100*inst[ln]/ti:5.1f}% thr {t:4.1f} L{ln:>4} | {src[ln-1].strip()[:100] if ln else ''}")
if len(sys.argv) > 4:  # ranges "name:a-b,name:a-b"
    for part in sys.argv[4].split(","):
        nm, ab = part.split(":"); a, b = map(int, ab.split("-"))
        s = sum(v for k, v in samp.items() if k and a <= k <= b); i = sum(v for k, v in inst.items() if k and a <= k <= b)
        t = sum(v for k, v in thr.items() if k and a <= k <= b)
        print(f"{nm:10s} samples {100*s/ts:5.1f}%  inst {100*i/ti:5.1f}%  thr/inst {t/max(i,1):4.1f}")
