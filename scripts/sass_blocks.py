"""Split one kernel's SASS (cuobjdump text) at a marker instruction and print block sizes.
   python scripts/sass_blocks.py /tmp/x.sass MANGLED_SUBSTR MARKER_REGEX"""
import re, sys
txt = open(sys.argv[1]).read().split("\n")
fn, marker = sys.argv[2], re.compile(sys.argv[3])
on, body = False, []
for line in txt:
    if line.strip().startswith("Function :"):
        on = fn in line
        continue
    if on and re.search(r"/\*[0-9a-f]{4,}\*/", line):
        body.append(line)
print("instructions:", len(body))
idx = [i for i, l in enumerate(body) if marker.search(l)]
print("markers at:", idx[:40])
print("gaps:", [b - a for a, b in zip(idx, idx[1:])][:40])
for k in ("STL", "LDL", "ATOMS", "BAR.SYNC", "IMAD.MOV", "S2R", "S2UR"):
    print(k, sum(1 for l in body if re.search(r"\b" + re.escape(k) + r"\b", l)))
