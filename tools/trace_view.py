"""Print the debug-64 pipeline trace of cluster 0 (k_quad_tc.cu), times relative to the MMA's full-wait."""
import sys

EV = ["tmaE", "tmaI", "ptop", "sgl", "emp", "lds", "sts", "fence", "sfull", "arr", "mfull", "commit", "mtop", "mfnc",
      "relay", "mful1"]
d = {}
for line in open(sys.argv[1]):
    if line.startswith("TR "):
        v = line.split()
        d[(int(v[1]), int(v[2]))] = [int(x) for x in v[3:]]
lo, hi = (int(sys.argv[2]), int(sys.argv[3])) if len(sys.argv) > 3 else (40, 60)
print("step  dt   | " + " ".join(f"{e:>6s}" for e in EV) + " || follower " + " ".join(f"{e:>6s}" for e in EV[:10]))
for s in range(lo, hi):
    L, F = d[(0, s)], d[(1, s)]
    base = L[10]
    f = lambda x: x - base if x else 0
    print(f"{s:3d} {L[10] - d[(0, s - 1)][10]:5d} | " + " ".join(f"{f(x):6d}" for x in L) + " || " +
          " ".join(f"{f(x):6d}" for x in F[:10]) + f" relay {f(F[14]):6d}")
