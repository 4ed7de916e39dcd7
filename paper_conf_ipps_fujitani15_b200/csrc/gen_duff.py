#!/usr/bin/env python3
"""Emit duff_pass.cuh: the fused multiword update X <- rshift(X - alpha*Y) of
PAPER.md §IV (L233, L237: one least- to most-significant pass, every word of X
and Y read once and every word of X written once), as straight-line sm_100a
code with a computed entry point.

Numbers live in registers, "top-aligned" per warp: word i of every lane's
operand sits in register s + i, where s = W - L and L is the warp-uniform
maximum operand length (euclid.cuh).  The pass must therefore start at the
dynamic (warp-uniform) register s and run to the static top W-1.  A `switch`
on s jumps to a per-entry head block (first limb: product, subtract without
borrow-in, r = ctz(z_s)) which then falls into the shared unrolled body chain
at limb s+1.  One indirect branch per pass, no per-limb length checks.

Per limb k of the body (SASS on sm_100a):
    IMAD.WIDE.U32  p = alpha*Y[k] + h        (product chain, carry h = hi(p))
    IADD3.X        z_k = X[k] - lo(p) - borrow   (PTX subc.cc chain)
    SHF.R.W        X[k-1] = funnel(z_{k-1}, z_k, r)  (rshift, L37)
plus the register-pair shuffle ptxas needs for the 64-bit addend.

Limb forms (template argument F of duff_pass, `form_code`):
    split  IMAD.WIDE.U32 (zero addend), IADD3 carry-add, IMAD.X, IADD3.X, SHF.R.W:
           three ALU-pipe and two FMA-pipe instructions per limb;
    wide   IMAD.WIDE.U32 with the 64-bit addend {h, 0} (PTX mul.wide + shr + add.s64),
           IMAD.MOV (pair shuffle), IADD3.X, SHF.R.W: the carry-add moves to the FMA pipe;
    mixM   every M-th limb split, the others wide.  The all-pairs kernel's ALU pipe is the
           busiest unit (ncu: 72.7 % against 55 % fmaheavy on cfg3), so mix2 balances the two:
           cfg3 240.9 -> 233.3 ms, cfg6 82.0 -> 80.7 ms (wide 238.7, mix3 237.7, mix4 238.6).

Run:  python gen_duff.py  (writes duff_pass.cuh next to this file)
"""
import os

WIDTHS = (16, 32, 64)


def form_code(form: str) -> int:
    """duff_pass's third template argument: 0 split, 1 wide, M >= 2 mixM."""
    if form == "split":
        return 0
    if form == "wide":
        return 1
    assert form.startswith("mix") and int(form[3:]) >= 2, form
    return int(form[3:])


def emit(W: int, form: str = "split", G: int = 1) -> str:
    """The whole pass as one inline-PTX block.

    Why PTX: written in C++, the computed entry (goto into a chain) is
    "structured" by the compiler, which interleaves the entry blocks with the
    chain and leaves a taken branch after every limb.  In PTX, `brx.idx`
    jumps to per-entry head blocks E_k that are laid out together and leave
    through a (always-true) predicated branch into the contiguous chain B_k,
    so the hot chain is straight-line code.

    Operands: %0 = r (out), %1 = z_s (out), %2..%(W+1) = X[k] (in/out),
    %(W+2)..%(2W+1) = Y[k], %(2W+2) = alpha, %(2W+3) = s.
    """
    FCODE = form_code(form)
    xa = lambda k: "%%%d" % (2 + k)
    ya = lambda k: "%%%d" % (W + 2 + k)
    al = "%%%d" % (2 * W + 2)
    sa = "%%%d" % (2 * W + 3)
    a = ["{", ".reg .u32 zp, z, lo, hi, t;", ".reg .u64 p, q, m;", ".reg .pred pe;",
         "setp.ge.s32 pe, %s, 0;" % sa,
         "ts: .branchtargets %s;" % ", ".join("E%d" % k for k in range(W)),
         "brx.idx %s, ts;" % sa]
    def limb(k):  # body limb k >= 1: product with carry, borrow chain, funnel shift into X[k-1]
        # "mixM": every M-th limb split, the rest wide (balances the ALU and FMA pipes)
        wide = form == "wide" or (form.startswith("mix") and k % int(form[3:]) != 0)
        if wide:  # 64-bit addend: IMAD.WIDE.U32 + pair shuffle (product chain on the FMA pipe)
            out = ["mul.wide.u32 m, %s, %s;" % (al, ya(k)),
                   "shr.u64 q, p, 32;",
                   "add.s64 p, m, q;",
                   "mov.b64 {lo, hi}, p;"]
        else:  # split: IMAD.WIDE + 32-bit add-with-carry of the high half
            out = ["mov.b64 q, {hi, 0};",
                   "mad.wide.u32 p, %s, %s, q;" % (al, ya(k)),
                   "mov.b64 {lo, hi}, p;"]
        return out + ["subc.cc.u32 z, %s, lo;" % xa(k),
                      "shf.r.wrap.b32 %s, zp, z, %%0;" % xa(k - 1),
                      "mov.u32 zp, z;"]

    def block_end(k):  # first limb after the G-aligned block that contains k
        return (k // G + 1) * G

    for k in range(W):
        e = min(block_end(k), W)
        nxt = "B%d" % e if e < W else "TOP"
        a += ["E%d:" % k,
              "mul.wide.u32 p, %s, %s;" % (al, ya(k)),
              "mov.b64 {lo, hi}, p;",
              "sub.cc.u32 zp, %s, lo;" % xa(k),
              "mov.u32 %1, zp;",
              "brev.b32 t, zp;",
              "clz.b32 %0, t;"]
        for j in range(k + 1, e):  # rest of the head's G-block, straight-line (no label inside)
            a += limb(j)
        a.append("@pe bra %s;" % nxt)
    a.append("bra.uni TOP;")
    for k in range(1, W):
        if k % G == 0:
            a.append("B%d:" % k)
        a += limb(k)
    a += ["TOP:", "shf.r.wrap.b32 %s, zp, 0, %%0;" % xa(W - 1), "}"]
    body = "\\n\\t".join(x.replace('"', '\\"') for x in a)
    outs = ['"=r"(r)', '"=r"(zs)'] + ['"+r"(X[%d])' % k for k in range(W)]
    ins = ['"r"(Y[%d])' % k for k in range(W)] + ['"r"(alpha)', '"r"(s)']
    o = ["template <>",
         "__device__ __forceinline__ uint32_t duff_pass<%d, %d, %d>(uint32_t (&X)[%d], const uint32_t (&Y)[%d], "
         "uint32_t alpha, int s, uint32_t &r) {" % (W, G, FCODE, W, W),
         "  uint32_t zs;",
         '  asm volatile("%s"' % body,
         "      : %s" % ", ".join(outs),
         "      : %s);" % ", ".join(ins),
         "  return zs;",
         "}"]
    return "\n".join(o)


def emit_cmpl(W: int, G: int, ones: bool) -> str:
    """Complement form (round 2): one operand of the pair is kept bit-complemented, so
    the update is a pure multiply-accumulate  T = X + alpha*Y + cin  (mod D^n, n = W - s)
    and the subtract-with-borrow chain of the split form disappears:
      * A-type (ones=True): X holds ~X0, Y plain, cin = 0:  T = D^n - 1 - (X0 - alpha*Y),
        so the complemented result is T >> r with ones shifted in at the top, r = ctz(~t_s);
      * B-type (ones=False): X plain, Y holds ~Y0, cin = alpha:  T = X - alpha*Y0 (mod D^n,
        exact since 0 <= X - alpha*Y0 < D^n), zeros shifted in, r = ctz(t_s).
    Per limb t_k + D c_k = alpha*y_k + x_k + c_{k-1} < 2^64, written as one 64-bit
    mad.wide plus one 64-bit add, which ptxas lowers to IMAD.WIDE.U32 + a three-input
    IADD3 (two carry-outs) + IADD3.X (two carry-ins): 4 instructions per limb with the
    funnel shift, against 5 for the split form (tools/limbmix2.cu: 8.8 vs 9.5 SMSP-cycles).

    Operands: %0 = r (out), %1 = t_s (out), %2..%(W+1) = X[k] (in/out),
    %(W+2)..%(2W+1) = Y[k], %(2W+2) = alpha, %(2W+3) = s, %(2W+4) = cin."""
    xa = lambda k: "%%%d" % (2 + k)
    ya = lambda k: "%%%d" % (W + 2 + k)
    al = "%%%d" % (2 * W + 2)
    sa = "%%%d" % (2 * W + 3)
    ci = "%%%d" % (2 * W + 4)
    a = ["{", ".reg .u32 tp, t, c, u;", ".reg .u64 p, q, w;", ".reg .pred pe;",
         "setp.ge.s32 pe, %s, 0;" % sa,
         "ts: .branchtargets %s;" % ", ".join("E%d" % k for k in range(W)),
         "brx.idx %s, ts;" % sa]

    def mac(k, cin, dst):
        return ["cvt.u64.u32 q, %s;" % xa(k),
                "mad.wide.u32 p, %s, %s, q;" % (al, ya(k)),
                "cvt.u64.u32 w, %s;" % cin,
                "add.u64 p, p, w;",
                "mov.b64 {%s, c}, p;" % dst]

    def limb(k):
        return mac(k, "c", "t") + ["shf.r.wrap.b32 %s, tp, t, %%0;" % xa(k - 1), "mov.u32 tp, t;"]

    for k in range(W):
        e = min((k // G + 1) * G, W)
        nxt = "B%d" % e if e < W else "TOP"
        a += ["E%d:" % k] + mac(k, ci, "tp") + ["mov.u32 %1, tp;"]
        a += (["not.b32 u, tp;", "brev.b32 u, u;"] if ones else ["brev.b32 u, tp;"]) + ["clz.b32 %0, u;"]
        for j in range(k + 1, e):
            a += limb(j)
        a.append("@pe bra %s;" % nxt)
    a.append("bra.uni TOP;")
    for k in range(1, W):
        if k % G == 0:
            a.append("B%d:" % k)
        a += limb(k)
    a += ["TOP:", "shf.r.wrap.b32 %s, tp, %s, %%0;" % (xa(W - 1), "0xffffffff" if ones else "0"), "}"]
    body = "\\n\\t".join(x.replace('"', '\\"') for x in a)
    outs = ['"=r"(r)', '"=r"(ts)'] + ['"+r"(X[%d])' % k for k in range(W)]
    ins = ['"r"(Y[%d])' % k for k in range(W)] + ['"r"(alpha)', '"r"(s)', '"r"(cin)']
    o = ["template <>",
         "__device__ __forceinline__ uint32_t duff_cpass<%d, %d, %s>(uint32_t (&X)[%d], const uint32_t (&Y)[%d], "
         "uint32_t alpha, uint32_t cin, int s, uint32_t &r) {" % (W, G, "true" if ones else "false", W, W),
         "  uint32_t ts;",
         '  asm volatile("%s"' % body,
         "      : %s" % ", ".join(outs),
         "      : %s);" % ", ".join(ins),
         "  return ts;",
         "}"]
    return "\n".join(o)


def emit_hybrid(W: int, G: int, side: str, form: str = "split") -> str:
    """Hybrid passes of the 4096-bit all-pairs kernel (kernels.cuh allpairs_hybrid_kernel):
    operand A lives in registers (top-aligned like every register kernel: word i at
    register s + i), operand B in shared memory, least significant word first, one row of
    32 lanes per word; with base = (B's row 0 address) - 128 s, B's word at register
    position k is at [base + 128 k] -- a static immediate per limb, and realigning A
    (s += 1) is a change of base, B never moves.
      side "A": A <- rshift(A - alpha*B), B read from shared memory;
      side "B": B <- rshift(B - alpha*A), B read and written in shared memory.
    Split form per limb (IMAD.WIDE carry addend, subc.cc borrow chain, funnel shift), G-limb
    blocks behind a brx.idx jump table on s, like emit().

    Operands: %0 = r (out), %1 = z_s (out), %2..%(W+1) = A[k] (side A: in/out, side B: in),
    %(W+2) = alpha, %(W+3) = s, %(W+4) = base (32-bit shared address)."""
    av = lambda k: "%%%d" % (2 + k)
    al = "%%%d" % (W + 2)
    sa = "%%%d" % (W + 3)
    ba = "%%%d" % (W + 4)
    K = lambda k: 128 * k
    a = ["{", ".reg .u32 zp, z, lo, hi, t, v, w;", ".reg .u64 p, q, m;", ".reg .pred pe;",
         "setp.ge.s32 pe, %s, 0;" % sa,
         "ts: .branchtargets %s;" % ", ".join("E%d" % k for k in range(W)),
         "brx.idx %s, ts;" % sa]

    def ldv(k):  # the shared-memory operand's word at register position k -> v
        return ["ld.shared.u32 v, [%s+%d];" % (ba, K(k))]

    def product(k):  # p = alpha * (multiplicand word k) + carry, split or wide (emit's forms)
        mw = "v" if side == "A" else av(k)
        if form == "wide" or (form.startswith("mix") and k % int(form[3:]) != 0):
            return ["mul.wide.u32 m, %s, %s;" % (al, mw), "shr.u64 q, p, 32;", "add.s64 p, m, q;",
                    "mov.b64 {lo, hi}, p;"]
        return ["mov.b64 q, {hi, 0};", "mad.wide.u32 p, %s, %s, q;" % (al, mw), "mov.b64 {lo, hi}, p;"]

    def limb(k):
        out = ldv(k) + product(k)
        if side == "A":
            out += ["subc.cc.u32 z, %s, lo;" % av(k),
                    "shf.r.wrap.b32 %s, zp, z, %%0;" % av(k - 1)]
        else:
            out += ["subc.cc.u32 z, v, lo;",
                    "shf.r.wrap.b32 w, zp, z, %0;",
                    "st.shared.u32 [%s+%d], w;" % (ba, K(k - 1))]
        return out + ["mov.u32 zp, z;"]

    for k in range(W):
        e = min((k // G + 1) * G, W)
        nxt = "B%d" % e if e < W else "TOP"
        a += ["E%d:" % k] + ldv(k)
        if side == "A":
            a += ["mul.wide.u32 p, %s, v;" % al, "mov.b64 {lo, hi}, p;", "sub.cc.u32 zp, %s, lo;" % av(k)]
        else:
            a += ["mul.wide.u32 p, %s, %s;" % (al, av(k)), "mov.b64 {lo, hi}, p;", "sub.cc.u32 zp, v, lo;"]
        a += ["mov.u32 %1, zp;", "brev.b32 t, zp;", "clz.b32 %0, t;"]
        for j in range(k + 1, e):
            a += limb(j)
        a.append("@pe bra %s;" % nxt)
    a.append("bra.uni TOP;")
    for k in range(1, W):
        if k % G == 0:
            a.append("B%d:" % k)
        a += limb(k)
    if side == "A":
        a += ["TOP:", "shf.r.wrap.b32 %s, zp, 0, %%0;" % av(W - 1), "}"]
    else:
        a += ["TOP:", "shf.r.wrap.b32 w, zp, 0, %0;", "st.shared.u32 [%s+%d], w;" % (ba, K(W - 1)), "}"]
    body = "\\n\\t".join(x.replace('"', '\\"') for x in a)
    if side == "A":
        outs = ['"=r"(r)', '"=r"(zs)'] + ['"+r"(A[%d])' % k for k in range(W)]
        ins = ['"r"(alpha)', '"r"(s)', '"r"(base)']
        sig = "uint32_t (&A)[%d]" % W
    else:
        outs = ['"=r"(r)', '"=r"(zs)']
        ins = ['"r"(A[%d])' % k for k in range(W)] + ['"r"(alpha)', '"r"(s)', '"r"(base)']
        sig = "uint32_t (&A)[%d]" % W  # read only (asm inputs)
    o = ["template <>",
         "__device__ __forceinline__ uint32_t duff_hpass<%d, %d, '%s'>(%s, uint32_t alpha, int s, uint32_t base, "
         "uint32_t &r) {" % (W, G, side, sig),
         "  uint32_t zs;",
         '  asm volatile("%s"' % body,
         "      : %s" % ", ".join(outs),
         "      : %s" % ", ".join(ins),
         '      : "memory");',
         "  return zs;",
         "}"]
    return "\n".join(o)


def main():
    import sys
    # Pass form per kernel family (measured on cfg3 / 2^20 1024-bit pairs, tools/ab_cfg3.sh):
    #   all-pairs + RSA-mode pairs, W <= 32: mix2 (every other limb with the 64-bit IMAD.WIDE addend:
    #     half the limbs move their carry-add from the ALU to the FMA pipe): cfg3 240.9 -> 234.2 ms,
    #     RSA pairs 2.73 -> 2.69 ms (wide 238.7 / 2.82, mix4 238.6 / 2.80);
    #   exact-mode pairs: split (mix2 3.85 -> 3.94 ms);  W = 64: split (all pairs use the complement form).
    form = sys.argv[1] if len(sys.argv) > 1 else os.environ.get("BULKGCD_PASS_FORM", "mix2")
    form64 = os.environ.get("BULKGCD_PASS_FORM64", "split")
    formx = os.environ.get("BULKGCD_PASS_FORM_EXACT", "split")
    # 4096-bit hybrid passes: mix2 (cfg8 5,563 -> 5,219 ms, cfg7 5.9 -> 5.5 ms)
    formh = os.environ.get("BULKGCD_PASS_FORM_HYBRID", "mix2")
    # W = 32 blocks of 8 limbs once the all-pairs loop carried two pass copies (cfg3 231.7 -> 230.0 ms;
    # 6: 230.8, 16: 271.9, 2: 240.7); W = 16 keeps 4 (its own knob below)
    G = int(os.environ.get("BULKGCD_PASS_G", "8"))
    # Exact-mode pairs kernel: G = 2 (cfg2 2^20 exact pairs 4.20 -> 3.87 ms; its larger
    # code -- Case-1 tail, L41 normalisation -- misses the i-cache at G = 4).  G = 2 for
    # the all-pairs kernel costs 246.7 -> 250.7 ms on cfg3, G = 8: 247.3 ms (exact 4.99).
    # Exact at G = 1: 3.98 ms (2048-bit 3.74), G = 3: 4.00 ms (3.58), against 3.87 / 3.46 at G = 2.
    GX = int(os.environ.get("BULKGCD_PASS_G_EXACT", "2"))
    G64 = int(os.environ.get("BULKGCD_PASS_G64", "2"))  # W = 64 has its own knob
    GR = int(os.environ.get("BULKGCD_PASS_G_RSA", "4"))  # RSA-mode pairs kernel, W <= 32
    G16 = int(os.environ.get("BULKGCD_PASS_G16", "4"))  # W = 16 at G = 2: cfg6 82.6 -> 83.4 ms, 8: 79.1 -> 79.2
    here = os.path.dirname(os.path.abspath(__file__))
    fw = lambda W: form64 if W >= 64 else form
    parts = [
        "// GENERATED by gen_duff.py -- do not edit by hand.",
        "// Fused X <- rshift(X - alpha*Y) limb pass with a computed entry (see gen_duff.py).",
        "#pragma once",
        "#include <cstdint>",
        "",
        "namespace bulkgcd {",
        "",
        "__device__ __forceinline__ uint32_t ctz32(uint32_t x) { return __clz(__brev(x)); }",
        "",
        "// Returns z_s (the lowest word of X - alpha*Y); r = ctz(z_s) (32 if z_s == 0, in which",
        "// case the funnel shifts wrap to 0 and X holds X - alpha*Y unshifted).",
        "// G = limbs per straight-line block of the chain (one predicated branch per block);",
        "// F = limb form (gen_duff.form_code: 0 split, 1 wide, M >= 2 every M-th limb split).",
        "template <int W, int G, int F>",
        "__device__ __forceinline__ uint32_t duff_pass(uint32_t (&X)[W], const uint32_t (&Y)[W], uint32_t alpha, int s,",
        "                                              uint32_t &r);",
        "",
        "// all-pairs and RSA-mode pairs kernels; W = 64 takes 2-limb blocks (cfg4 900.7 -> 898.4 ms,",
        "// 2^18 2048-bit RSA pairs 2.89 -> 2.81 ms; 8-limb blocks: 1,135 ms)",
        "template <int W>",
        "constexpr int PASS_G = W >= 64 ? %d : (W <= 16 ? %d : %d);" % (G64, G16, G),
        "template <int W>",
        "constexpr int PASS_F = W >= 64 ? %d : %d;  // %s / %s" % (form_code(form64), form_code(form), form64, form),
        "// RSA-mode pairs kernel (one-entry loop): 4-limb blocks at W <= 32 (2^20 pairs 2.46 ms against 3.14 at 8)",
        "template <int W>",
        "constexpr int PASS_G_RSA = W >= 64 ? %d : %d;" % (G64, GR),
        "constexpr int PASS_G_EXACT = %d;  // exact-mode pairs kernel (smaller code: i-cache)" % GX,
        "constexpr int PASS_F_EXACT = %d;  // %s" % (form_code(formx), formx),
        "",
    ]
    parts += [
        "// Complement form (emit_cmpl): T = X + alpha*Y + cin (mod D^n); ONES: shift ones in at the",
        "// top and r = ctz(~t_s) (X holds a complemented operand).  Returns t_s.",
        "template <int W, int G, bool ONES>",
        "__device__ __forceinline__ uint32_t duff_cpass(uint32_t (&X)[W], const uint32_t (&Y)[W], uint32_t alpha,",
        "                                               uint32_t cin, int s, uint32_t &r);",
        "",
    ]
    GH = int(os.environ.get("BULKGCD_PASS_G_HYBRID", "4"))
    parts += [
        "// Hybrid passes (emit_hybrid): A in registers, B in shared memory at [base + 128 k].",
        "template <int W, int G, char SIDE, class AR>",
        "__device__ __forceinline__ uint32_t duff_hpass(AR &A, uint32_t alpha, int s, uint32_t base, uint32_t &r);",
        "constexpr int PASS_G_HYBRID = %d;" % GH,
        "",
        emit_hybrid(128, GH, "A", formh), "",
        emit_hybrid(128, GH, "B", formh), "",
    ]
    for W in WIDTHS:
        gw = G64 if W >= 64 else (G16 if W <= 16 else G)
        gr = G64 if W >= 64 else GR
        for g, f in sorted({(gw, fw(W)), (gr, fw(W)), (GX, formx)}):
            parts.append(emit(W, f, g))
            parts.append("")
        for ones in (True, False):
            parts.append(emit_cmpl(W, gw, ones))
            parts.append("")
    parts.append("}  // namespace bulkgcd")
    out = os.environ.get("BULKGCD_DUFF_OUT", os.path.join(here, "duff_pass.cuh"))
    with open(out, "w") as f:
        f.write("\n".join(parts) + "\n")


if __name__ == "__main__":
    main()
