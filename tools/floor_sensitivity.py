"""Sensitivity of the library rule to its TLP floor (min_warps_sm), R27 on, over every stored sweep."""
import sys, math
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tools")
import rule_replay as rr
orig = rr.rule_hw
for fl in (6, 8, 10, 12, 16):
    def hwf(name, fl=fl):
        h = orig("b200"); h.min_warps_sm = fl; return h
    rr.rule_hw = hwf
    res = rr.replay("x", ["final", "heldout", "heldout2", "heldout3", "heldout4", "heldout5", "heldout6", "heldout7", "heldout8", "partition"], False)
    q = [x[5] for x in res]
    cont = [x for x in res if x[6] > 1.05]
    print(f"floor {fl:2d}: within5 {sum(1 for v in q if v <= 1.05)}/{len(q)} geomean {math.exp(sum(map(math.log, q))/len(q)):.4f} worst {max(q):.3f}  over-full(contended) {math.exp(sum(math.log(x[6]/x[5]) for x in cont)/len(cont)):.3f}")
