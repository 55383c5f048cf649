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
              143: "upd done", 144: "upd scan", 148: "u0 entry", 149: "u1 scanned",
              150: "u2 bnd", 151: "u3 end", 152: "u4 ret", 154: "kmax(warp)", 155: "lanes rmin-clock<=8",
              156: "b0 done", 157: "b1 issued", 158: "b1 done", 159: "b2 issued", 160: "b2 done", 161: "b3 issued",
              162: "b3 done", 163: "b4 issued", 164: "b4 done"})
names.update({160: "U entry", 161: "U fastdone", 162: "U b0 start", 163: "U b0 done", 164: "U b1 start", 165: "U b1 done",
              166: "U b2 start", 167: "U b2 done", 168: "U b3 start", 169: "U b3 done", 170: "U b4 start", 171: "U b4 done",
              172: "U scanned", 175: "kmax"})

d = collections.defaultdict(dict)
spans = collections.defaultdict(dict)   # kernel -> cta -> (entry, after wait, end, tiles) [globaltimer ns]
for line in open(sys.argv[1]):
    if line.startswith("cta "):
        _, k, c, e0, e1, e2, e3 = line.split()
        spans[int(k)][int(c)] = (int(e0), int(e1), int(e2), int(e3))
        continue
    t, slot, v = map(int, line.split())
    d[t][slot] = v
for lo, hi, title in ((0, 128, "conv_stack"), (128, 256, "fc1_head")):
    VALS = (154, 155, 175)   # plain values, not timestamps
    vals = [v for t in d for sl, v in d[t].items() if lo <= sl < hi and sl not in VALS]
    if not vals:
        continue
    base = min(vals)
    print(f"== {title}")
    for t in sorted(d):
        ev = sorted((v - base, names.get(sl, str(sl))) for sl, v in d[t].items() if lo <= sl < hi and sl not in VALS)
        extra = "  ".join(f"{names[sl]}={d[t][sl]}" for sl in VALS if sl in d[t] and lo <= sl < hi)
        print(f" tile {t}: " + "  ".join(f"{n}={v}" for v, n in ev) + ("  | " + extra if extra else ""))

if spans:
    # per-CTA spans of two consecutive steps (kernels 0/1: conv_stack / fc1_head of step s,
    # 2/3: of step s + 1), ns relative to the first conv_stack entry of step s
    base = min(v[0] for v in spans[0].values())
    kn = {0: "conv_stack s", 1: "fc1_head s", 2: "conv_stack s+1", 3: "fc1_head s+1"}
    print("== per-CTA spans (ns from the first conv_stack entry of step s)")
    for k in sorted(spans):
        rows = spans[k]
        ent = sorted(v[0] - base for v in rows.values())
        wt = sorted(v[1] - base for v in rows.values())
        end = sorted(v[2] - base for v in rows.values())
        last = max(rows, key=lambda c: rows[c][2])
        tiles = collections.Counter((v[3] >> 8) if k % 2 else v[3] for v in rows.values())
        print(f" {kn[k]:15s} CTAs {len(rows):3d}  entry {ent[0]:7d}..{ent[-1]:7d}  wait-return {wt[0]:7d}..{wt[-1]:7d}"
              f"  end p50 {end[len(end) // 2]:7d} p90 {end[int(len(end) * 0.9)]:7d} max {end[-1]:7d} (CTA {last},"
              f" tiles {rows[last][3] >> 8 if k % 2 else rows[last][3]}{', Pmax ' + str(rows[last][3] & 255) if k % 2 else ''})"
              f"  tiles/CTA {dict(sorted(tiles.items()))}")
    if 1 in spans:
        pm = collections.Counter(v[3] & 255 for v in spans[1].values())
        bypm = collections.defaultdict(list)
        for v in spans[1].values():
            bypm[v[3] & 255].append(v[2] - v[1])
        print(" fc1_head s: Pmax of a CTA's tiles -> CTAs, mean (end - wait-return) ns:",
              {p: (pm[p], int(sum(bypm[p]) / len(bypm[p]))) for p in sorted(pm)})
