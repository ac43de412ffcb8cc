"""Aggregate an ncu 'cuda,sass' source CSV by CUDA source line: share of executed
instructions and of warp-stall samples (top N lines)."""
import csv, sys, collections
path = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
rows = list(csv.reader(open(path)))
f = None; hdr = None; inst = collections.Counter(); stall = collections.Counter(); text = {}
for r in rows:
    if r and r[0] == "File Path": f = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No": hdr = r; continue
    if not hdr or not r or not r[0].isdigit(): continue
    key = (f, int(r[0])); text[key] = r[1]
    o = len(r) - len(hdr)          # source text containing commas may shift columns
    try:
        inst[key] += int(r[7 + o] or 0); stall[key] += int(r[4 + o] or 0)
    except ValueError:
        pass
ti = sum(inst.values()) or 1; ts = sum(stall.values()) or 1
print(f"total inst {ti}, stall samples {ts}")
for k, v in sorted(inst.items(), key=lambda t: -(t[1] / ti + stall[t[0]] / ts))[:top]:
    print(f"{100*v/ti:5.1f}%i {100*stall[k]/ts:5.1f}%s {k[0]}:{k[1]:<4} {text[k][:90]}")
