"""Summarise `ncu -i X --page source --csv --print-source cuda,sass -k K`: per source line stall samples + instructions."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = None; out = []
for r in rows:
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and len(r) == len(hdr) and r[0]:
        try: s = int(r[4] or 0); ie = int(r[7] or 0)
        except ValueError: continue
        out.append((s, r[0], ie, r[1][:120]))
tot = sum(o[0] for o in out) or 1
itot = sum(o[2] for o in out) or 1
print(f"total samples {tot}  warp-instructions {itot:.3e}")
for s, ln, ie, src in sorted(out, reverse=True)[:n]:
    print(f"{100*s/tot:5.1f}% L{ln:>4} inst={100*ie/itot:5.1f}% | {src.strip()}")
