"""Generates paper_conf_middleware_hafeezsg021_b200/csrc/fast_walk_ptx.inc: the eval32 search
walk's uniform segment (D = 2, two candidates per lane, uint32 time; DESIGN.md §3.4 "fast walk")
as one inline-PTX loop with `brx.idx.uni` jump tables.  With two candidates per lane (uint32)
the lane's two values of a slot sit side by side (eval32.cu kInterleave2), so every ring,
staging and cold access of the pair is one 8-byte access (cold-slot reductions stay 4-byte).

Outside its group's special positions (the region and the producers of region ops, the
Layout::spec_pos lists) every lane of a warp has the base device of every op and successor, so a
step's whole control path -- begin on device xu or a continuation step, then per edge: link or
not, register / ring / cold slot, first push or max -- is a function of (xu, class, cross) of its
<= 2 edges.  The loop runs steps until a limit address (the tile's end, the swapped pair, or
the first step of the next special position, which the caller looks up in op_off32) and
dispatches each step through two warp-uniform jump tables:
  TA[(continuation << 5) | k0]  begin (first steps) + edge 0
  TB[k1]                        edge 1
with k = yu | class << 1 | xu << 4 read from the step head (StepHead.kinds, one byte per slot,
kept by the layout, K4 and the swap patch); the handler knows cross = (yu != xu); class 0 far,
1 far first, 2 near, 3 near first, 4 next, 5 empty slot (layout_format.h).  Same arithmetic as eval32.cu's C++ step
(PAPER.md L142-146, L188-198): C_v = min(max(r, dev_free[xu]) + p_v, SAT); a crossing edge
A = min(max(C_v, link_free[xu -> 1-xu]) + t, SAT), link_free = A; else A = C_v.

usage: python scripts/gen_fast_walk.py  (rewrites the .inc; commit both)
"""
import os

HERE = os.path.dirname(os.path.abspath(__file__))
OUT = os.path.join(HERE, "..", "paper_conf_middleware_hafeezsg021_b200", "csrc", "fast_walk_ptx.inc")

SAT = "0xF0000000"


def operands(cpl, wide):
    """read-write %0 sp, %1 v, then per candidate c: d0[c], d1[c], l01[c], l10[c], fwd[c],
    nfar[c], nnear[c] (each group of cpl consecutive); inputs lim (the step address where the
    segment must stop: the tile's end, the swapped pair or the first step of the next special
    position), ring, stage (shared u32), cold (global u64).  wide: the exact 64-bit instance."""
    global SP, V, D, L, FWD, NFAR, NNEAR, LIM, RING, STAGE, COLD, CPL, W, TY, TB_, CB, IL
    CPL, W = cpl, wide
    IL = cpl == 2 and not wide          # a lane's two candidates side by side (8 bytes per slot)
    TY = "u64" if wide else "u32"       # time type
    TB_ = 8 if wide else 4              # bytes per time value
    CB = 32 * TB_                       # bytes of one 32-lane column
    k = iter(range(2, 2 + 7 * cpl + 4))
    grp = lambda: tuple(f"%{next(k)}" for _ in range(cpl))   # noqa: E731
    SP, V = "%0", "%1"
    D = (grp(), grp())
    L = (grp(), grp())                 # l01 (xu 0 -> 1), l10 (xu 1 -> 0)
    FWD, NFAR, NNEAR = grp(), grp(), grp()
    LIM, RING, STAGE, COLD = (f"%{next(k)}" for _ in range(4))


def tadd(dst, a, dur):
    """dst = a + dur, saturated at SAT for uint32 (every duration < 2^28 so it never wraps),
    exact for uint64; dur is a u32 record field"""
    if W:
        return [f"cvt.u64.u32 z, {dur};", f"add.u64 {dst}, {a}, z;"]
    return [f"add.u32 {dst}, {a}, {dur};", f"min.u32 {dst}, {dst}, {SAT};"]


def log2(x):
    return x.bit_length() - 1


def edge(xu, cls, cross, rec):
    """PTX of one uniform edge (record registers rec = (t0, succ, target, t1))."""
    if cls == 5:
        return []
    C = D[xu]
    out = []
    if cross:
        t = rec[3] if xu else rec[0]
        for c in range(CPL):
            out += [f"max.{TY} w{c}, {C[c]}, {L[xu][c]};"] + tadd(f"w{c}", f"w{c}", t) + \
                   [f"mov.{TY} {L[xu][c]}, w{c};"]
        a = ("w0", "w1")[:CPL]
    else:
        a = C
    if cls == 4:
        out += [f"max.{TY} {FWD[c]}, {FWD[c]}, {a[c]};" for c in range(CPL)]
        return out
    # slot byte offset of the lane's column: (target & mask) x CPL x sizeof(T)/4 (the records
    # hold offsets of 4-byte columns)
    sh = log2(CPL * TB_ // 4)
    out += [f"and.b32 o, {rec[2]}, 0x1FFFFFFF;"] + ([f"shl.b32 o, o, {sh};"] if sh else [])
    if cls in (2, 3):
        out += [f"add.u32 s, {RING}, o;"]
        if IL:                          # both candidates with one 8-byte access
            if cls == 2:
                out += ["ld.shared.v2.u32 {y0, y1}, [s];", f"max.u32 y0, y0, {a[0]};",
                        f"max.u32 y1, y1, {a[1]};", "st.shared.v2.u32 [s], {y0, y1};"]
            else:
                out += [f"st.shared.v2.u32 [s], {{{a[0]}, {a[1]}}};"]
            return out
        for c in range(CPL):
            if cls == 2:
                out += [f"ld.shared.{TY} y{c}, [s+{CB * c}];", f"max.{TY} y{c}, y{c}, {a[c]};",
                        f"st.shared.{TY} [s+{CB * c}], y{c};"]
            else:
                out += [f"st.shared.{TY} [s+{CB * c}], {a[c]};"]
    else:
        out += ["cvt.u64.u32 g, o;", f"add.u64 g, {COLD}, g;"]
        if IL and cls == 1:
            return out + [f"st.global.v2.u32 [g], {{{a[0]}, {a[1]}}};"]
        for c in range(CPL):
            co = 4 * c if IL else CB * c
            if cls == 1:
                out += [f"st.global.{TY} [g+{co}], {a[c]};"]
            else:
                out += [f"red.relaxed.gpu.global.max.{TY} [g+{co}], {a[c]};"]
    return out


def begin(xu):
    """C_v = min(max(r, dev_free[xu]) + p, SAT); dev_free[xu] = C_v (arrivals in r0/r1)."""
    out = []
    for c in range(CPL):
        out += [f"max.{TY} w{c}, r{c}, {D[xu][c]};"] + tadd(D[xu][c], f"w{c}", "h0")
    return out


def segment(cpl, wide=False, ra=False, dt=False, early=False, ce=False, ks=False):
    """ks: edge 1's table entry is extracted from the head inside the edge-0 handlers, after the
    slot-1-empty test (77% of steps have no edge 1), instead of at the loop top.
    ce (two candidates per lane, uint32): the far-arrival copy is one 16-byte cp.async.cg by
    every even lane (its own and its odd neighbour's pair) instead of an 8-byte cp.async.ca by
    every lane.
    ra: the next step's head is read one step ahead (its kinds feed the jump-table load
    before the current step's work; 4 register moves per step).  dt: direct threading -- every
    handler ends with its own copy of the loop's top (limit check, record loads, first-step
    work, dispatch), so no join point sits inside the loop (ptxas otherwise brackets every
    iteration with a reconvergence barrier and sends it through one far-away join block).
    early (with dt): each edge-0 handler loads the next step's head as soon as the begin has
    used p_v, so the head's latency overlaps the handler and the tail does not reload it"""
    operands(cpl, wide)
    cb = CB * cpl                       # bytes of one ring slot (cpl columns of 32 lanes)
    sh = log2(cb)
    A = ("a0", "a1", "a2", "a3")
    B = ("b0", "b1", "b2", "b3")
    ta = [f"FA{i}" for i in range(64)]
    tb = [f"FB{i}" for i in range(32)]
    P = []
    P += ["{",
          ".reg .pred p, q, q2;",
          ".reg .u32 h0, h1, h2, h3, a0, a1, a2, a3, b0, b1, b2, b3, t, k0, k1, o, s, sz;",
          f".reg .{TY} r0, r1, w0, w1, y0, y1;",
          ".reg .u64 g, z;",
          "TA: .branchtargets " + ", ".join(ta) + ";",
          "TB: .branchtargets " + ", ".join(tb) + ";"]
    if ce:
        P += [".reg .pred pe;", "mov.u32 t, %laneid;", "and.b32 t, t, 1;", "setp.eq.u32 pe, t, 0;"]
    if ra:
        P += [".reg .u32 n0, n1, n2, n3;",
              f"ld.shared.v4.u32 {{n0, n1, n2, n3}}, [{SP}];"]

    def top(tag, have_head=False):
        """the loop's top: stop at the limit, load the step, first-step work, dispatch TA"""
        T = [f"setp.ge.u32 p, {SP}, {LIM};",
             "@p bra.uni FDONE;"]
        if have_head:           # loaded early by the handler (the tile is padded by one step)
            pass
        elif ra:                # the tile is padded by one step: [sp + 48] is always readable
            T += ["mov.u32 h0, n0;", "mov.u32 h1, n1;", "mov.u32 h2, n2;", "mov.u32 h3, n3;",
                  f"ld.shared.v4.u32 {{n0, n1, n2, n3}}, [{SP}+48];"]
        else:
            T += [f"ld.shared.v4.u32 {{h0, h1, h2, h3}}, [{SP}];"]
        T += [f"ld.shared.v4.u32 {{a0, a1, a2, a3}}, [{SP}+16];",
              f"ld.shared.v4.u32 {{b0, b1, b2, b3}}, [{SP}+32];",
              # the slots' jump-table entries, kept by the layout / K4 / swap patches
              # (StepHead.kinds: yu | class << 1 | xu << 4 per slot byte)
              "and.b32 k0, h1, 31;"]
        if not ks:
            T += ["shr.u32 k1, h1, 8;",
                  "and.b32 k1, k1, 31;"]
        T += [
              "and.b32 t, h1, 0xE00;",
              "setp.eq.u32 q2, t, 0xA00;",            # slot 1 empty (class 5): no TB dispatch
              "and.b32 t, h3, 16;",
              "setp.ne.u32 q, t, 0;",
              f"@q bra.uni FCONT{tag};",
              # first step of the op at v + 1 (the caller's limit stops the loop at the first
              # step of the next special position, so every first step here is a uniform op)
              f"add.u32 {V}, {V}, 1;",
              # far arrivals of v + 11 -> staging ring (zero-filled without a far producer)
              f"add.u32 t, {V}, 11;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
              f"add.u32 s, {STAGE}, t;",
              "setp.ge.s32 p, h2, 0;", "max.s32 t, h2, 0;", f"mul.wide.u32 g, t, {cb};",
              f"add.u64 g, {COLD}, g;", f"selp.u32 sz, {(16 if ce else 8) if IL else TB_}, 0, p;"]
        if IL and ce:
            T += ["@pe cp.async.cg.shared.global [s], [g], 16, sz;"]
        elif IL:
            T += ["cp.async.ca.shared.global [s], [g], 8, sz;"]
        else:
            T += [f"cp.async.ca.shared.global [s+{CB * c}], [g+{CB * c}], {TB_}, sz;"
                  for c in range(cpl)]
        T += ["cp.async.commit_group;",
              "cp.async.wait_group 10;",
              # arrivals of v: staged far, forwarded (distance 1), near ring when flagged
              "and.b32 t, h3, 8;", "setp.ne.u32 p, t, 0;"]
        for c in range(cpl):
            T += [f"selp.{TY} r{c}, {NNEAR[c]}, 0, p;", f"max.{TY} r{c}, r{c}, {NFAR[c]};",
                  f"max.{TY} r{c}, r{c}, {FWD[c]};"]
        # read ahead the far / near arrivals of v + 1 (final once v starts)
        T += [f"add.u32 t, {V}, 1;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
              f"add.u32 s, {STAGE}, t;"]
        if IL:
            T += [f"ld.shared.v2.u32 {{{NFAR[0]}, {NFAR[1]}}}, [s];", f"add.u32 s, {RING}, t;",
                  f"ld.shared.v2.u32 {{{NNEAR[0]}, {NNEAR[1]}}}, [s];"]
        else:
            T += [f"ld.shared.{TY} {NFAR[c]}, [s+{CB * c}];" for c in range(cpl)]
            T += [f"add.u32 s, {RING}, t;"]
            T += [f"ld.shared.{TY} {NNEAR[c]}, [s+{CB * c}];" for c in range(cpl)]
        T += [f"mov.{TY} {FWD[c]}, 0;" for c in range(cpl)]
        T += ["brx.idx.uni k0, TA;",
              f"FCONT{tag}:",
              "add.u32 k0, k0, 32;",
              "brx.idx.uni k0, TA;"]
        return T

    def tail(tag):
        if dt:
            return [f"add.u32 {SP}, {SP}, 48;"] + top(tag, have_head=early)
        return ["bra.uni FNEXT;"]

    if dt:
        P += top("")
    else:
        P += ["FLOOP:"] + top("")

    def decode(e):                      # table entry -> (xu, class, cross)
        yu, cls, xu = e & 1, (e >> 1) & 7, (e >> 4) & 1
        return xu, cls, int(yu != xu)

    for i in range(64):
        cont, e = i >> 5, i & 31
        xu, cls, cross = decode(e)
        P.append(f"FA{i}:")
        if cls > 5:                     # unused entries (class codes 6, 7)
            P.append("bra.uni FDONE;")
            continue
        if not cont:
            P += begin(xu)
        if dt and early:        # p_v used: the next step's head may replace this one
            P += [f"ld.shared.v4.u32 {{h0, h1, h2, h3}}, [{SP}+48];"]
        P += edge(xu, cls, cross, A)
        if dt:
            P += [f"@q2 bra.uni FTA{i};", "brx.idx.uni k1, TB;", f"FTA{i}:"] + tail(f"A{i}")
        else:
            P += ["@q2 bra.uni FNEXT;"]
            if ks:
                P += ["shr.u32 k1, h1, 8;", "and.b32 k1, k1, 31;"]
            P += ["brx.idx.uni k1, TB;"]
    for i in range(32):
        xu, cls, cross = decode(i)
        P.append(f"FB{i}:")
        if cls > 5:
            P.append("bra.uni FDONE;")
            continue
        P += edge(xu, cls, cross, B)
        if dt:
            P += tail(f"B{i}")
        elif i < 31:
            P.append("bra.uni FNEXT;")
    if not dt:
        P += ["FNEXT:", f"add.u32 {SP}, {SP}, 48;", "bra.uni FLOOP;"]
    P += ["FDONE:", "}"]
    return P


def segment_d4(cpl):
    """D = 3..4 (two plane bits per code), uint32 time, state in shared memory (eval32.cu
    SmemState32: device columns at dst + x * slot, links at lst + (x * 4 + y) * slot; a slot is 32
    lanes x cpl, a lane's pair side by side for cpl 2).  The jump tables dispatch on the edge's
    (class, crossing) only -- 12 entries; the device and link columns are addressed at run time
    from the slot's kinds byte (yu | class << 2 | xu << 5; D <= 4), the link class of x -> y is
    bit x * 4 + y of cls4.  (A table specialised on (xu, yu, class) -- 256 + 128 entries -- ran
    slower than the C++ walk: the handlers no longer fit the instruction cache.)"""
    global CPL
    CPL = cpl
    IL2 = cpl == 2
    SLOT = 128 * cpl                    # bytes of a state column / ring slot
    sh = log2(SLOT)
    k = iter(range(2, 2 + 3 * cpl + 7))
    grp = lambda: tuple(f"%{next(k)}" for _ in range(cpl))   # noqa: E731
    SP_, V_ = "%0", "%1"
    FWD_, NFAR_, NNEAR_ = grp(), grp(), grp()
    LIM_, RING_, STAGE_, COLD_, DST_, LST_, CLS_ = (f"%{next(k)}" for _ in range(7))

    def lds2(dst, addr):
        if IL2:
            return [f"ld.shared.v2.u32 {{{dst[0]}, {dst[1]}}}, [{addr}];"]
        return [f"ld.shared.u32 {dst[0]}, [{addr}];"]

    def sts2(addr, src):
        if IL2:
            return [f"st.shared.v2.u32 [{addr}], {{{src[0]}, {src[1]}}};"]
        return [f"st.shared.u32 [{addr}], {src[0]};"]

    C = ("c0", "c1")[:cpl]
    W_ = ("w0", "w1")[:cpl]
    Y = ("y0", "y1")[:cpl]

    def edge4(cls, cross, rec, lk):
        """lk: register holding x * 4 + y of this edge's link (crossing edges)"""
        if cls == 5:
            return []
        out = []
        if cross:                       # FCFS link xu -> yu: its class picks t0 / t1
            out += [f"shr.u32 t, {CLS_}, {lk};", "and.b32 t, t, 1;", "setp.ne.u32 p, t, 0;",
                    f"selp.u32 t, {rec[3]}, {rec[0]}, p;", f"mad.lo.u32 s, {lk}, {SLOT}, {LST_};"]
            out += lds2(W_, "s")
            for c in range(cpl):
                out += [f"max.u32 {W_[c]}, {W_[c]}, {C[c]};", f"add.u32 {W_[c]}, {W_[c]}, t;",
                        f"min.u32 {W_[c]}, {W_[c]}, {SAT};"]
            out += sts2("s", W_)
            a = W_
        else:
            a = C
        if cls == 4:
            return out + [f"max.u32 {FWD_[c]}, {FWD_[c]}, {a[c]};" for c in range(cpl)]
        out += [f"and.b32 o, {rec[2]}, 0x1FFFFFFF;"] + (["shl.b32 o, o, 1;"] if cpl == 2 else [])
        if cls in (2, 3):
            out += [f"add.u32 s, {RING_}, o;"]
            if cls == 2:
                out += lds2(Y, "s")
                out += [f"max.u32 {Y[c]}, {Y[c]}, {a[c]};" for c in range(cpl)]
                out += sts2("s", Y)
            else:
                out += sts2("s", a)
        else:
            out += ["cvt.u64.u32 g, o;", f"add.u64 g, {COLD_}, g;"]
            if cls == 1:
                if IL2:
                    out += [f"st.global.v2.u32 [g], {{{a[0]}, {a[1]}}};"]
                else:
                    out += [f"st.global.u32 [g], {a[0]};"]
            else:
                out += [f"red.relaxed.gpu.global.max.u32 [g+{4 * c}], {a[c]};" for c in range(cpl)]
        return out

    def kind(byte_shift, k, lk):
        """k = class * 2 + (yu != xu), lk = xu * 4 + yu, from the slot's kinds byte"""
        return [f"shr.u32 t, h1, {byte_shift};",
                "and.b32 u, t, 3;",                       # yu
                "shr.u32 xx, t, 5;", "and.b32 xx, xx, 3;", # xu
                f"shl.b32 {lk}, xx, 2;", f"or.b32 {lk}, {lk}, u;",
                "setp.ne.u32 p, u, xx;", "selp.u32 u, 1, 0, p;",
                f"shr.u32 {k}, t, 1;", f"and.b32 {k}, {k}, 14;", f"or.b32 {k}, {k}, u;"]

    A = ("a0", "a1", "a2", "a3")
    B = ("b0", "b1", "b2", "b3")
    ta = [f"FA{i}" for i in range(32)]
    tb = [f"FB{i}" for i in range(16)]
    P = ["{",
         ".reg .pred p, q, q2;",
         ".reg .u32 h0, h1, h2, h3, a0, a1, a2, a3, b0, b1, b2, b3, t, u, xx, k0, k1, l0, l1, "
         "o, s, sz, r0, r1, w0, w1, y0, y1, c0, c1;",
         ".reg .u64 g;",
         "TA: .branchtargets " + ", ".join(ta) + ";",
         "TB: .branchtargets " + ", ".join(tb) + ";",
         "FLOOP:",
         f"setp.ge.u32 p, {SP_}, {LIM_};",
         "@p bra.uni FDONE;",
         f"ld.shared.v4.u32 {{h0, h1, h2, h3}}, [{SP_}];",
         f"ld.shared.v4.u32 {{a0, a1, a2, a3}}, [{SP_}+16];",
         f"ld.shared.v4.u32 {{b0, b1, b2, b3}}, [{SP_}+32];"]
    P += kind(0, "k0", "l0") + kind(8, "k1", "l1")
    P += ["setp.ge.u32 q2, k1, 10;",          # slot 1 empty (class 5): no TB dispatch
          "and.b32 t, h3, 16;",
          "setp.ne.u32 q, t, 0;",
          # the op's device column (xu of slot 0 = the op's base code)
          "shr.u32 t, l0, 2;", f"mad.lo.u32 xx, t, {SLOT}, {DST_};",
          "@q bra.uni FCONT;",
          f"add.u32 {V_}, {V_}, 1;",
          f"add.u32 t, {V_}, 11;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
          f"add.u32 s, {STAGE_}, t;",
          "setp.ge.s32 p, h2, 0;", "max.s32 t, h2, 0;", f"mul.wide.u32 g, t, {SLOT};",
          f"add.u64 g, {COLD_}, g;", f"selp.u32 sz, {4 * cpl}, 0, p;",
          f"cp.async.ca.shared.global [s], [g], {4 * cpl}, sz;",
          "cp.async.commit_group;",
          "cp.async.wait_group 10;",
          "and.b32 t, h3, 8;", "setp.ne.u32 p, t, 0;"]
    for c in range(cpl):
        P += [f"selp.u32 r{c}, {NNEAR_[c]}, 0, p;", f"max.u32 r{c}, r{c}, {NFAR_[c]};",
              f"max.u32 r{c}, r{c}, {FWD_[c]};"]
    P += [f"add.u32 t, {V_}, 1;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
          f"add.u32 s, {STAGE_}, t;"]
    P += lds2(NFAR_, "s")
    P += [f"add.u32 s, {RING_}, t;"]
    P += lds2(NNEAR_, "s")
    P += [f"mov.u32 {FWD_[c]}, 0;" for c in range(cpl)]
    # C_v = min(max(r, dev_free[xu]) + p, SAT), dev_free[xu] = C_v
    P += lds2(W_, "xx")
    for c in range(cpl):
        P += [f"max.u32 {C[c]}, r{c}, {W_[c]};", f"add.u32 {C[c]}, {C[c]}, h0;",
              f"min.u32 {C[c]}, {C[c]}, {SAT};"]
    P += sts2("xx", C)
    P += ["brx.idx.uni k0, TA;",
          "FCONT:"]                     # a continuation: dev_free[xu] still holds C_v
    P += lds2(C, "xx")
    P += ["add.u32 k0, k0, 16;",
          "brx.idx.uni k0, TA;"]
    for i in range(32):
        e = i & 15
        cls, cross = e >> 1, e & 1
        P.append(f"FA{i}:")
        if cls > 5:
            P.append("bra.uni FDONE;")
            continue
        P += edge4(cls, cross, A, "l0")
        P += ["@q2 bra.uni FNEXT;", "brx.idx.uni k1, TB;"]
    for i in range(16):
        cls, cross = i >> 1, i & 1
        P.append(f"FB{i}:")
        if cls <= 5:
            P += edge4(cls, cross, B, "l1")
        if i < 15:
            P.append("bra.uni FNEXT;")
    P += ["FNEXT:", f"add.u32 {SP_}, {SP_}, 48;", "bra.uni FLOOP;", "FDONE:", "}"]
    return P


def segment_rows(cpl, pf=0, v2=False, ra=False, win=False, fold=False, foldx=False):
    """foldx (with fold): the op-word window switch rides on the dispatch too -- bit 4 of the
    edge-0 index = "this op is the last of its 32-op window" (first steps only); entries 16-23
    switch the op-word window, 48-55 both windows, then continue in the normal handler.
    fold (with win): the successor-word window switch rides on the step's dispatch -- the
    edge-0 table index carries bit 5 = "this step's slots are in the next window" and those 16
    entries switch the window, redo the step's two shuffles and continue in the normal handler --
    instead of an if-converted block that ptxas executes (predicated) on every step.
    win (with v2): both word streams are read 32 words at a time -- lane l loads word
    base + l with one coalesced load, the next window is loaded a window ahead (out of line, once
    per 32 ops / 16 steps) and a step takes its words with warp shuffles, so no step waits on a
    global load (ra's register read-ahead was undone by ptxas, which copied the loaded word into
    the loop-carried register before the dispatch and so waited for it there).
    ra (with v2): the successor words of the next step and the op word of the next op are
    loaded one step / one op ahead into registers (re-primed at every segment entry; the
    workspace pads both streams so the last step's read-ahead stays in bounds) -- the L1 hit
    rate of these uniform loads is ~13% behind the cold-slot traffic, so a load issued at its
    use waited on L2.
    v2: the op's register holds its raw 32-row word and the lane tests it with a lane mask
    (one LOP3 to a predicate instead of shift, and, compare), and a crossing edge updates its
    link with two predicated selects instead of predicate ANDs and moves.
    pf > 0: each step also prefetches into L1 the successor-word stream pf bytes ahead and
    the op-word stream pf/2 bytes ahead (both advance one 32-bit word per slot / per op), so
    the step's uniform loads hit L1 instead of waiting on L2 once every 16-32 steps.
    Explicit rows (eval32 mode 0), D = 2, uint32 time: every lane has its own devices (K5's
    bit-sliced words: the op's word at xb + 4v, the successors' at yb + 4·slot, bit `lane`), so
    the device and link choices are per-lane selects, but the control -- first step or not, the
    edge's class -- is the step's and dispatches through 8-entry jump tables."""
    global CPL
    CPL = cpl
    IL2 = cpl == 2
    SLOT = 128 * cpl
    sh = log2(SLOT)
    k = iter(range(3, 3 + 8 * cpl + 5 + 2 * cpl))
    grp = lambda: tuple(f"%{next(k)}" for _ in range(cpl))   # noqa: E731
    SP_, V_, YS_ = "%0", "%1", "%2"
    D0_, D1_, L01_, L10_, FWD_, NFAR_, NNEAR_, X_ = (grp() for _ in range(8))
    LIM_, RING_, STAGE_, COLD_, LANE_ = (f"%{next(k)}" for _ in range(5))
    XB_, YB_ = grp(), grp()
    C = ("c0", "c1")[:cpl]
    PX = ("px0", "px1")[:cpl]

    def lds2(dst, addr):
        if IL2:
            return [f"ld.shared.v2.u32 {{{dst[0]}, {dst[1]}}}, [{addr}];"]
        return [f"ld.shared.u32 {dst[0]}, [{addr}];"]

    def sts2(addr, src):
        if IL2:
            return [f"st.shared.v2.u32 [{addr}], {{{src[0]}, {src[1]}}};"]
        return [f"st.shared.u32 [{addr}], {src[0]};"]

    def edge_rows(cls, rec, ywreg):
        if cls == 5:
            return []
        out = []
        a = ("w0", "w1")[:cpl]
        for c in range(cpl):
            if v2:
                out += [f"xor.b32 t, {ywreg[c]}, {X_[c]};", "and.b32 t, t, lm;",
                        "setp.ne.u32 pc, t, 0;",                                      # crossing
                        f"selp.u32 u, {L10_[c]}, {L01_[c]}, {PX[c]};",
                        f"selp.u32 tt, {rec[3]}, {rec[0]}, {PX[c]};",
                        f"max.u32 u, u, {C[c]};", "add.u32 u, u, tt;", f"min.u32 u, u, {SAT};",
                        f"@pc selp.u32 {L10_[c]}, u, {L10_[c]}, {PX[c]};",
                        f"@pc selp.u32 {L01_[c]}, {L01_[c]}, u, {PX[c]};",
                        f"selp.u32 {a[c]}, u, {C[c]}, pc;"]
                continue
            out += [f"shr.u32 t, {ywreg[c]}, {LANE_};", "and.b32 t, t, 1;",
                    f"xor.b32 t, t, {X_[c]};", "setp.ne.u32 pc, t, 0;",             # crossing
                    f"selp.u32 u, {L10_[c]}, {L01_[c]}, {PX[c]};",
                    f"selp.u32 tt, {rec[3]}, {rec[0]}, {PX[c]};",
                    f"max.u32 u, u, {C[c]};", "add.u32 u, u, tt;", f"min.u32 u, u, {SAT};",
                    f"and.pred pq, pc, {PX[c]};", f"@pq mov.u32 {L10_[c]}, u;",
                    f"and.pred pq, pc, !{PX[c]};", f"@pq mov.u32 {L01_[c]}, u;",
                    f"selp.u32 {a[c]}, u, {C[c]}, pc;"]
        if cls == 4:
            return out + [f"max.u32 {FWD_[c]}, {FWD_[c]}, {a[c]};" for c in range(cpl)]
        out += [f"and.b32 o, {rec[2]}, 0x1FFFFFFF;"] + (["shl.b32 o, o, 1;"] if cpl == 2 else [])
        if cls in (2, 3):
            out += [f"add.u32 s, {RING_}, o;"]
            if cls == 2:
                Y = ("y0", "y1")[:cpl]
                out += lds2(Y, "s")
                out += [f"max.u32 {Y[c]}, {Y[c]}, {a[c]};" for c in range(cpl)]
                out += sts2("s", Y)
            else:
                out += sts2("s", a)
        else:
            out += ["cvt.u64.u32 g, o;", f"add.u64 g, {COLD_}, g;"]
            if cls == 1:
                out += ([f"st.global.v2.u32 [g], {{{a[0]}, {a[1]}}};"] if IL2
                        else [f"st.global.u32 [g], {a[0]};"])
            else:
                out += [f"red.relaxed.gpu.global.max.u32 [g+{4 * c}], {a[c]};" for c in range(cpl)]
        return out

    A = ("a0", "a1", "a2", "a3")
    B = ("b0", "b1", "b2", "b3")
    YA = ("ya0", "ya1")[:cpl]           # slot-0 successor words per candidate group
    YBw = ("yb0", "yb1")[:cpl]          # slot-1
    ta = [f"FA{i}" for i in range(16)]
    if foldx:                           # 16-23 op-word switch, 32-47 successor-word switch,
        ta += ([f"FX{i}" for i in range(8)] + ["FDONE"] * 8 +      # 48-55 both
               [f"FS{i}" for i in range(16)] + [f"FSX{i}" for i in range(8)] + ["FDONE"] * 8)
    elif fold:                          # entries 32-47: window switch, then FA{i}
        ta += ["FDONE"] * 16 + [f"FS{i}" for i in range(16)]
    tb = [f"FB{i}" for i in range(8)]
    P = ["{",
         ".reg .pred p, q, q2, pc, pq, px0, px1;",
         ".reg .u32 h0, h1, h2, h3, a0, a1, a2, a3, b0, b1, b2, b3, t, u, tt, k0, k1, o, s, sz, "
         "r0, r1, w0, w1, y0, y1, c0, c1, ya0, ya1, yb0, yb1, xw, lm;",
         ".reg .u64 g, gy;",
         "TA: .branchtargets " + ", ".join(ta) + ";",
         "TB: .branchtargets " + ", ".join(tb) + ";"]
    YAn = ("yan0", "yan1")[:cpl]
    YBn = ("ybn0", "ybn1")[:cpl]
    XN = ("xn0", "xn1")[:cpl]
    if ra:
        P += [".reg .u32 yan0, yan1, ybn0, ybn1, xn0, xn1;"]
        for c in range(cpl):
            P += [f"mul.wide.u32 gy, {YS_}, 4;", f"add.u64 gy, {YB_[c]}, gy;",
                  f"ld.global.nc.v2.u32 {{{YAn[c]}, {YBn[c]}}}, [gy];",
                  f"add.u32 t, {V_}, 1;", "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {XB_[c]}, gy;",
                  f"ld.global.nc.u32 {XN[c]}, [gy];"]
    XWC, XWN = ("xwc0", "xwc1")[:cpl], ("xwn0", "xwn1")[:cpl]
    YWC, YWN = ("ywc0", "ywc1")[:cpl], ("ywn0", "ywn1")[:cpl]
    if win:
        P += [".reg .u32 xwc0, xwc1, xwn0, xwn1, ywc0, ywc1, ywn0, ywn1, xwb, ywb, ix, iy, sw;",
              f"add.u32 xwb, {V_}, 1;", "and.b32 xwb, xwb, -32;",
              f"and.b32 ywb, {YS_}, -32;"]
        for c in range(cpl):
            P += [f"add.u32 t, xwb, {LANE_};", "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {XB_[c]}, gy;",
                  f"ld.global.nc.u32 {XWC[c]}, [gy];", f"ld.global.nc.u32 {XWN[c]}, [gy+128];",
                  f"add.u32 t, ywb, {LANE_};", "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {YB_[c]}, gy;",
                  f"ld.global.nc.u32 {YWC[c]}, [gy];", f"ld.global.nc.u32 {YWN[c]}, [gy+128];"]
    if v2:
        P += [f"shl.b32 lm, 1, {LANE_};"]
    P += ["FLOOP:",
         f"setp.ge.u32 p, {SP_}, {LIM_};",
         "@p bra.uni FDONE;",
         f"ld.shared.v4.u32 {{h0, h1, h2, h3}}, [{SP_}];",
         f"ld.shared.v4.u32 {{a0, a1, a2, a3}}, [{SP_}+16];",
         f"ld.shared.v4.u32 {{b0, b1, b2, b3}}, [{SP_}+32];"]
    if fold:                            # shuffles from the current window; a step whose
        # slots lie in the next one (iy >= 32) redoes them in its FS entry after the switch
        P += [f"sub.u32 iy, {YS_}, ywb;", "and.b32 sw, iy, 32;"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {YA[c]}, {YWC[c]}, iy, 31, -1;"]
        P += ["add.u32 t, iy, 1;"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {YBw[c]}, {YWC[c]}, t, 31, -1;"]
    elif win:                           # this step's two slots: shuffles from the window
        P += [f"sub.u32 ix, {YS_}, ywb;", "setp.ge.u32 p, ix, 32;", "@p bra.uni FYW;", "FYR:"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {YA[c]}, {YWC[c]}, ix, 31, -1;"]
        P += ["add.u32 ix, ix, 1;"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {YBw[c]}, {YWC[c]}, ix, 31, -1;"]
    for c in range(cpl if not win else 0):   # both slots' successor words of candidate group c
        if ra:
            P += [f"mov.u32 {YA[c]}, {YAn[c]};", f"mov.u32 {YBw[c]}, {YBn[c]};",
                  f"mul.wide.u32 gy, {YS_}, 4;", f"add.u64 gy, {YB_[c]}, gy;",
                  f"ld.global.nc.v2.u32 {{{YAn[c]}, {YBn[c]}}}, [gy+8];"]
            continue
        P += [f"mul.wide.u32 gy, {YS_}, 4;", f"add.u64 gy, {YB_[c]}, gy;",
              f"ld.global.nc.v2.u32 {{{YA[c]}, {YBw[c]}}}, [gy];"]
        if pf:
            P += [f"prefetch.global.L1 [gy+{pf}];"]
    P += [f"add.u32 {YS_}, {YS_}, 2;",
          "shr.u32 k0, h1, 1;", "and.b32 k0, k0, 7;"]
    if fold:
        P += ["or.b32 k0, k0, sw;"]
    P += [
          "shr.u32 k1, h1, 9;", "and.b32 k1, k1, 7;",
          "setp.eq.u32 q2, k1, 5;",             # slot 1 empty: no TB dispatch
          "and.b32 t, h3, 16;",
          "setp.ne.u32 q, t, 0;",
          "@q bra.uni FCONT;",
          f"add.u32 {V_}, {V_}, 1;"]
    if foldx:                           # ix < 32: the switch ran at the window's last op
        P += [f"sub.u32 ix, {V_}, xwb;"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {X_[c]}, {XWC[c]}, ix, 31, -1;"]
        P += ["add.u32 t, ix, 1;", "shr.u32 t, t, 1;", "and.b32 t, t, 16;", "or.b32 k0, k0, t;"]
    elif win:
        P += [f"sub.u32 ix, {V_}, xwb;", "setp.ge.u32 p, ix, 32;", "@p bra.uni FXW;", "FXR:"]
        for c in range(cpl):
            P += [f"shfl.sync.idx.b32 {X_[c]}, {XWC[c]}, ix, 31, -1;"]
    for c in range(cpl if not win else 0):   # the op's device in each lane's row: bit `lane`
        if ra:
            P += [f"mov.u32 {X_[c]}, {XN[c]};", f"mul.wide.u32 gy, {V_}, 4;",
                  f"add.u64 gy, {XB_[c]}, gy;", f"ld.global.nc.u32 {XN[c]}, [gy+4];"]
            continue
        P += [f"mul.wide.u32 gy, {V_}, 4;", f"add.u64 gy, {XB_[c]}, gy;"]
        if v2:
            P += [f"ld.global.nc.u32 {X_[c]}, [gy];"]
        else:
            P += ["ld.global.nc.u32 xw, [gy];", f"shr.u32 xw, xw, {LANE_};", f"and.b32 {X_[c]}, xw, 1;"]
        if pf:
            P += [f"prefetch.global.L1 [gy+{pf // 2}];"]
    P += [f"add.u32 t, {V_}, 11;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
          f"add.u32 s, {STAGE_}, t;",
          "setp.ge.s32 p, h2, 0;", "max.s32 t, h2, 0;", f"mul.wide.u32 g, t, {SLOT};",
          f"add.u64 g, {COLD_}, g;", f"selp.u32 sz, {4 * cpl}, 0, p;",
          f"cp.async.ca.shared.global [s], [g], {4 * cpl}, sz;",
          "cp.async.commit_group;",
          "cp.async.wait_group 10;",
          "and.b32 t, h3, 8;", "setp.ne.u32 p, t, 0;"]
    for c in range(cpl):
        P += [f"selp.u32 r{c}, {NNEAR_[c]}, 0, p;", f"max.u32 r{c}, r{c}, {NFAR_[c]};",
              f"max.u32 r{c}, r{c}, {FWD_[c]};"]
    P += [f"add.u32 t, {V_}, 1;", "and.b32 t, t, 15;", f"shl.b32 t, t, {sh};",
          f"add.u32 s, {STAGE_}, t;"]
    P += lds2(NFAR_, "s")
    P += [f"add.u32 s, {RING_}, t;"]
    P += lds2(NNEAR_, "s")
    P += [f"mov.u32 {FWD_[c]}, 0;" for c in range(cpl)]
    # C_v = min(max(r, dev_free[x]) + p, SAT) per lane, dev_free[x] = C_v
    for c in range(cpl):
        P += ([f"and.b32 t, {X_[c]}, lm;", f"setp.ne.u32 {PX[c]}, t, 0;"] if v2 else
              [f"setp.ne.u32 {PX[c]}, {X_[c]}, 0;"])
        P += [f"selp.u32 t, {D1_[c]}, {D0_[c]}, {PX[c]};",
              f"max.u32 {C[c]}, r{c}, t;", f"add.u32 {C[c]}, {C[c]}, h0;",
              f"min.u32 {C[c]}, {C[c]}, {SAT};",
              f"@{PX[c]} mov.u32 {D1_[c]}, {C[c]};", f"@!{PX[c]} mov.u32 {D0_[c]}, {C[c]};"]
    P += ["brx.idx.uni k0, TA;",
          "FCONT:"]                     # a continuation: dev_free[x] still holds C_v
    for c in range(cpl):
        P += ([f"and.b32 t, {X_[c]}, lm;", f"setp.ne.u32 {PX[c]}, t, 0;"] if v2 else
              [f"setp.ne.u32 {PX[c]}, {X_[c]}, 0;"])
        P += [f"selp.u32 {C[c]}, {D1_[c]}, {D0_[c]}, {PX[c]};"]
    P += ["add.u32 k0, k0, 8;",
          "brx.idx.uni k0, TA;"]
    for i in range(16):
        cls = i & 7
        P.append(f"FA{i}:")
        if cls > 5:
            P.append("bra.uni FDONE;")
            continue
        P += edge_rows(cls, A, YA)
        P += ["@q2 bra.uni FNEXT;", "brx.idx.uni k1, TB;"]
    for i in range(8):
        P.append(f"FB{i}:")
        if i <= 5:
            P += edge_rows(i, B, YBw)
        if i < 7:
            P.append("bra.uni FNEXT;")
    P += ["FNEXT:", f"add.u32 {SP_}, {SP_}, 48;", "bra.uni FLOOP;"]
    def yswitch():
        out = ["add.u32 ywb, ywb, 32;"]
        for c in range(cpl):
            out += [f"mov.u32 {YWC[c]}, {YWN[c]};", f"add.u32 t, ywb, {LANE_};",
                    "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {YB_[c]}, gy;",
                    f"ld.global.nc.u32 {YWN[c]}, [gy+128];"]
        out += ["sub.u32 iy, iy, 32;"]
        for c in range(cpl):
            out += [f"shfl.sync.idx.b32 {YA[c]}, {YWC[c]}, iy, 31, -1;"]
        out += ["add.u32 t, iy, 1;"]
        for c in range(cpl):
            out += [f"shfl.sync.idx.b32 {YBw[c]}, {YWC[c]}, t, 31, -1;"]
        return out

    def xswitch():
        out = ["add.u32 xwb, xwb, 32;"]
        for c in range(cpl):
            out += [f"mov.u32 {XWC[c]}, {XWN[c]};", f"add.u32 t, xwb, {LANE_};",
                    "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {XB_[c]}, gy;",
                    f"ld.global.nc.u32 {XWN[c]}, [gy+128];"]
        return out

    if fold:                            # the successor-word window switch (entries 32-47)
        for i in range(16):
            P += [f"FS{i}:"] + yswitch() + [f"bra.uni FA{i};"]
    if foldx:                           # the op-word switch (16-23), both (48-55)
        for i in range(8):
            P += [f"FX{i}:"] + xswitch() + [f"bra.uni FA{i};"]
            P += [f"FSX{i}:"] + xswitch() + yswitch() + [f"bra.uni FA{i};"]
    if win and not fold:                # window switches, out of line
        P += ["FYW:", "add.u32 ywb, ywb, 32;"]
        for c in range(cpl):
            P += [f"mov.u32 {YWC[c]}, {YWN[c]};", f"add.u32 t, ywb, {LANE_};",
                  "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {YB_[c]}, gy;",
                  f"ld.global.nc.u32 {YWN[c]}, [gy+128];"]
        P += [f"sub.u32 ix, {YS_}, ywb;", "bra.uni FYR;"]
    if win and not foldx:
        P += ["FXW:", "add.u32 xwb, xwb, 32;"]
        for c in range(cpl):
            P += [f"mov.u32 {XWC[c]}, {XWN[c]};", f"add.u32 t, xwb, {LANE_};",
                  "mul.wide.u32 gy, t, 4;", f"add.u64 gy, {XB_[c]}, gy;",
                  f"ld.global.nc.u32 {XWN[c]}, [gy+128];"]
        P += [f"sub.u32 ix, {V_}, xwb;", "bra.uni FXR;"]
    P += ["FDONE:", "}"]
    return P


def main():
    with open(OUT, "w") as f:
        f.write("// generated by scripts/gen_fast_walk.py -- do not edit\n")
        f.write("// eval32.cu fast_segment (DESIGN.md §3.4 fast walk): uniform steps in one PTX loop\n")
        for cpl, wide, ra, dt, name in ((1, False, False, False, "1"), (2, False, False, False, "2"),
                                        (1, True, False, False, "1W"),
                                        (1, False, True, False, "1_RA"), (2, False, True, False, "2_RA"),
                                        (1, True, True, False, "1W_RA"),
                                        (1, False, False, True, "1_DT"), (2, False, False, True, "2_DT"),
                                        (1, True, False, True, "1W_DT")):
            P = segment(cpl, wide, ra, dt, early=dt)
            f.write(f"#define PESTO_FAST_WALK_PTX{name} \\\n" +
                    " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
            print(OUT, name, len(P), "PTX lines")
            if name != "2":
                continue
            name = "2_CE"
            P = segment(cpl, wide, ra, dt, early=dt, ce=True)
            f.write(f"#define PESTO_FAST_WALK_PTX{name} \\\n" +
                    " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
            print(OUT, name, len(P), "PTX lines")
            name = "2_CEKS"
            P = segment(cpl, wide, ra, dt, early=dt, ce=True, ks=True)
            f.write(f"#define PESTO_FAST_WALK_PTX{name} \\\n" +
                    " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
            print(OUT, name, len(P), "PTX lines")
        for cpl in (1, 2):
            for pf, v2, ra, suf in ((0, False, False, ""), (512, False, False, "_PF"),
                                    (0, True, False, "_V2"), (512, True, False, "_V2PF"),
                                    (0, True, True, "_V3")):
                P = segment_rows(cpl, pf, v2, ra)
                f.write(f"#define PESTO_FAST_ROWS_PTX{cpl}{suf} \\\n" +
                        " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
                print(OUT, f"{cpl}_ROWS{suf}", len(P), "PTX lines")
            for suf, fold, foldx in (("_V4", False, False), ("_V5", True, False),
                                     ("_V6", True, True)):
                P = segment_rows(cpl, 0, True, False, True, fold, foldx)
                f.write(f"#define PESTO_FAST_ROWS_PTX{cpl}{suf} \\\n" +
                        " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
                print(OUT, f"{cpl}_ROWS{suf}", len(P), "PTX lines")
        for cpl in (1, 2):
            P = segment_d4(cpl)
            f.write(f"#define PESTO_FAST_WALK_PTX{cpl}_D4 \\\n" +
                    " \\\n".join('    "' + l + '\\n"' for l in P) + "\n")
            print(OUT, f"{cpl}_D4", len(P), "PTX lines")


if __name__ == "__main__":
    main()
