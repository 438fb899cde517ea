"""Aggregate an ncu SASS source page (csv) per CUDA source line, using nvdisasm -g line info of the same cubin.

usage: python scripts/sass_lines.py <disasm -g output> <function substring> <ncu sass csv> [top]
"""
import csv, re, sys, collections
dis, fn, page = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
addr2line, cur_line, in_fn = {}, None, False
for ln in open(dis):
    m = re.match(r'\s*\.section\s+\.text\.(\S+?),', ln)
    if m:
        in_fn = fn in m.group(1)
        continue
    if not in_fn:
        continue
    m = re.search(r'## File ".*?", line (\d+)', ln)
    if m:
        cur_line = int(m.group(1))
        continue
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/', ln)
    if m and cur_line is not None:
        addr2line[int(m.group(1), 16)] = cur_line
rows = list(csv.reader(open(page)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hi]
ia, isamp, iinst = hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
base = None
for r in rows[hi + 1:]:
    if r and r[0].startswith("0x"):
        base = int(r[0], 16); break
agg = collections.defaultdict(lambda: [0.0, 0.0, collections.Counter()])
tot = [0.0, 0.0]
for r in rows[hi + 1:]:
    if len(r) <= iinst or not r[ia].startswith("0x") and not r[ia].isdigit():
        continue
    a = (int(r[ia], 16) - base) if r[ia].startswith("0x") else int(r[ia])
    line = addr2line.get(a, -1)
    s = float(r[isamp] or 0); n = float(r[iinst] or 0)
    agg[line][0] += s; agg[line][1] += n; tot[0] += s; tot[1] += n
    for i in stall_cols:
        v = float(r[i] or 0)
        if v: agg[line][2][hdr[i]] += v
src = open("/root/repo/paper_conf_ipps_wei024_b200/csrc/kernels.cu").read().splitlines()
print(f"total samples {tot[0]:.0f}  warp-instructions {tot[1]:.3e}  mapped addrs {len(addr2line)}")
for line, (s, n, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    txt = src[line - 1].strip()[:70] if line > 0 else "?"
    tops = ",".join(f"{k[6:]}:{v/s*100:.0f}" for k, v in st.most_common(3)) if s else ""
    print(f"{line:5d} {s/tot[0]*100:5.1f}% smp {n/tot[1]*100:5.1f}% inst  [{tops}]  {txt}")
