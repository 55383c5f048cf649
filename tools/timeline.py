"""Print the per-tile pipeline timeline of a PSIM_DEBUG_TIMING dump (libpsim built
with PSIM_TIMING=1): conv_stack slots 0..127, fc1_head slots 128..  (clock64 cycles
relative to the first event of each kernel, CTA 0, first 4 tiles)."""
import collections
import sys

names = {}
for j in range(4):
    names[0 + 2 * j] = f"c1({j})wait"; names[1 + 2 * j] = f"c1({j})go"
for h in range(2):
    for kh in range(2):
        names[8 + 2 * (h * 2 + kh)] = f"c2({h},{kh})wait"; names[9 + 2 * (h * 2 + kh)] = f"c2({h},{kh})go"
for kh in range(2):
    names[16 + 2 * kh] = f"c3({kh})wait"; names[17 + 2 * kh] = f"c3({kh})go"
for j in range(4):
    names[32 + 4 * j] = f"e1({j})wait"; names[33 + 4 * j] = f"e1({j})C1"; names[34 + 4 * j] = f"e1({j})ld"
    names[35 + 4 * j] = f"e1({j})A2free"; names[48 + j] = f"e1({j})done"
for h in range(2):
    names[56 + 4 * h] = f"e2({h})wait"; names[57 + 4 * h] = f"e2({h})C2"; names[58 + 4 * h] = f"e2({h})A3free"
    names[59 + 4 * h] = f"e2({h})done"
names.update({64: "e3wait", 65: "e3C3", 66: "e3done", 67: "e3staged", 68: "e3ld0", 69: "e3ld1", 80: "g start"})
for j in range(4):
    names[81 + 3 * j] = f"g{j}a"; names[82 + 3 * j] = f"g{j}slot"; names[83 + 3 * j] = f"g{j}built"
for j in range(4):
    names[96 + 2 * j] = f"g{j}issued"; names[97 + 2 * j] = f"g{j}ldq"
    names[104 + j] = f"g{j}rfull"
    names[112 + 3 * j] = f"g{j}sts"; names[113 + 3 * j] = f"g{j}fenced"; names[114 + 3 * j] = f"g{j}expect"
names.update({128: "tma start", 129: "tma end", 132: "mma wait tempty", 133: "mma start", 134: "mma issued",
              140: "epi start", 141: "epi F ready", 142: "epi y done", 145: "upd start", 146: "upd y ready",
              143: "upd done", 144: "upd scan"})

d = collections.defaultdict(dict)
for line in open(sys.argv[1]):
    t, slot, v = map(int, line.split())
    d[t][slot] = v
for lo, hi, title in ((0, 128, "conv_stack"), (128, 256, "fc1_head")):
    vals = [v for t in d for sl, v in d[t].items() if lo <= sl < hi]
    if not vals:
        continue
    base = min(vals)
    print(f"== {title}")
    for t in sorted(d):
        ev = sorted((v - base, names.get(sl, str(sl))) for sl, v in d[t].items() if lo <= sl < hi)
        print(f" tile {t}: " + "  ".join(f"{n}={v}" for v, n in ev))
