"""Offline model of the shared-memory wavefronts of tri_tiled_kernel (one
instance slot = LPI lanes).  Phases: LDS.32 -> 1 phase of 32 lanes, LDS.64 ->
2 of 16, LDS.128 -> 4 of 8; a phase costs max over bank groups of the number of
DISTINCT addresses mapping there (broadcast is free).  Used to compare table
layouts / schedules before spending GPU time; check against ncu's
l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld."""
import sys
from collections import defaultdict


def colbase(m):
    return 2 * m * m + 3 * m


def xc(a, m):
    return 4 * (colbase(m) + a)


def wavefronts(addrs, width):
    """addrs: {lane: word address} for active lanes; width in words (1, 2, 4)."""
    lanes_per_phase = 32 // width
    tot = 0
    phases = defaultdict(dict)
    for lane, a in addrs.items():
        phases[lane // lanes_per_phase][lane] = a
    for ph in phases.values():
        banks = defaultdict(set)
        for a in ph.values():
            banks[(a // width) % (32 // width)].add(a)
        tot += max(len(v) for v in banks.values())
    return tot


def split_log2(t, D, lpi):
    ls = 0
    while (2 << ls) * t <= lpi and (1 << ls) < D - 1:
        ls += 1
    return ls


def model(n=64, lpi=16, xcf=xc, verbose=False, qhigh=True, interleave=True):
    """Wavefronts per instance.  interleave: the kernel's LPI = 16 mapping,
    two instances on alternate lanes, tables 16 words (mod 32) apart."""
    NT = (n + 3) // 4
    words = 4 * colbase(NT)
    stride = words + ((16 - words) % 32) if interleave else words
    dense = fix = 0
    dense_ideal = 0
    for D in range(1, NT):
        ls = split_log2(NT - D, D, lpi)
        s = 1 << ls
        lanes = {}
        for lane in range(32 if lpi == 16 else lpi):
            slot, li = (lane & 1, lane >> 1) if (interleave and lpi == 16) else (lane // lpi, lane % lpi)
            if qhigh:       # kernel's mapping: tile index low bits, split index high bits
                ib = lpi.bit_length() - 1 - ls
                I, q = li & ((1 << ib) - 1), li >> ib
            else:
                I, q = li >> ls, li & (s - 1)
            if I < NT - D:
                lanes[lane] = (I, q, slot * stride)
        # dense iterations
        it = 0
        while True:
            act = {}
            for li, (I, q, b) in lanes.items():
                m = I + 1 + q + it * s
                if m < I + D:
                    act[li] = (I, m, I + D, b)
            if not act:
                break
            for u in range(4):
                dense += wavefronts({li: b + xcf(4 * I, m) + 4 * u for li, (I, m, J, b) in act.items()}, 4)
                dense += wavefronts({li: b + xcf(4 * m, J) + 4 * u for li, (I, m, J, b) in act.items()}, 4)
            dense_ideal += 8 * ((len(act) + 7) // 8)
            it += 1
        fl = {li: (I, b) for li, (I, q, b) in lanes.items() if q == 0}
        for r in range(4):
            if r < 3:
                fix += wavefronts({li: b + xcf(4 * I, I) + 4 * r for li, (I, b) in fl.items()}, 4)
                fix += wavefronts({li: b + xcf(4 * (I + D), I + D) + 4 * r for li, (I, b) in fl.items()}, 4)
            fix += 2 * wavefronts({li: b + xcf(4 * I, I + D) + 4 * r for li, (I, b) in fl.items()}, 4)   # ld + st
        if verbose:
            print(D, s, len(lanes), dense, fix)
    per = 2 if lpi == 16 else 1
    return dense / per, dense_ideal / per, fix / per


if __name__ == "__main__":
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
    for inter in (False, True):
        d, di, f = model(n, interleave=inter)
        print(f"n={n} interleave={inter}: dense {d} (phases {di}), fix-up ld+st {f} wavefronts per instance")
