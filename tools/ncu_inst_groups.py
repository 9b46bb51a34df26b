"""Instruction-count groups of an ncu report's SASS: executed warp-instructions grouped by the
execution count of each SASS line (a loop body shares one count), with each group's first lines."""
import collections, csv, io, subprocess, sys

rep = sys.argv[1]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
hdr, block = None, []
for r in csv.reader(io.StringIO(src)):
    if r and r[0] == "Address":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        block.append(r)
iex, isrc = hdr.index("Instructions Executed"), hdr.index("Source")
groups = collections.defaultdict(list)
for r in block:
    n = int(r[iex] or 0)
    if n:
        groups[n].append(r[isrc].strip())
tot = sum(n * len(v) for n, v in groups.items())
print(f"total {tot / 1e6:.1f} M warp-instructions")
for n, v in sorted(groups.items(), key=lambda kv: -kv[0] * len(kv[1]))[:int(sys.argv[2]) if len(sys.argv) > 2 else 15]:
    print(f"{n:>11} x {len(v):4d} = {n * len(v) / 1e6:8.1f} M ({100 * n * len(v) / tot:4.1f}%)  {' | '.join(v[:6])[:150]}")
