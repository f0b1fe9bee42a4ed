"""Three independent MSM routes for the oracle (test infrastructure only).

Q = sum_{i<n} k_i * P_i in E(F_p)   (§2.2)

* msm_naive        — each product k_i P_i by double-and-add PMUL,
                     summed with Formula (1).
* msm_pippenger    — plain Pippenger as PAPER.md §2.3 describes it:
                     ceil(λ/s) windows of s-bit UNSIGNED chunks m_i, bucket scatter into
                     2^s - 1 buckets, bucket-sum B_m, bucket-reduce W_j = sum_m m*B_m by the
                     running sum (2 PADD per bucket, the 2^(s+1) of PAPER.md:143),
                     window-reduce by Horner with s PDBL per window (λ PDBL in total).
                     Deliberately a different digit rule and coordinates than the GPU path.
* msm_closed_form  — for generated inputs P_i = e_i G: Q = (sum k_i e_i mod r) G
                     (linearity of the group law; pinned against the other two routes).
All return affine points (None = O).
"""
from . import ec


def msm_naive(ks, Ps, c):
    Q = None
    for k, P in zip(ks, Ps):
        Q = ec.add(Q, ec.mul(k, P, c), c)
    return Q


def msm_pippenger(ks, Ps, c, s=8):
    """PAPER.md:141-143, unsigned s-bit windows, affine arithmetic."""
    lam = c.lam
    nwin = -(-lam // s)               # ceil(λ/s)
    mask = (1 << s) - 1
    W = []
    for j in range(nwin):
        # bucket scatter + bucket-sum
        B = [None] * (1 << s)
        for k, P in zip(ks, Ps):
            m = (k >> (j * s)) & mask
            if m:
                B[m] = ec.add(B[m], P, c)
        # bucket-reduce: W_j = sum_m m * B_m via running sum from the top bucket
        running = None
        Wj = None
        for m in range(mask, 0, -1):
            running = ec.add(running, B[m], c)
            Wj = ec.add(Wj, running, c)
        W.append(Wj)
    # window-reduce (Horner): Q = W_{nwin-1}; Q = 2^s Q + W_j
    Q = None
    for j in range(nwin - 1, -1, -1):
        for _ in range(s):
            Q = ec.double(Q, c)
        Q = ec.add(Q, W[j], c)
    return Q


def msm_closed_form(ks, es, c):
    """Q = (sum k_i e_i mod r) * G for P_i = e_i * G."""
    t = 0
    for k, e in zip(ks, es):
        t += k * e
    return ec.mul(t % c.r, c.G, c)


def closed_form_arith(ks_sum: int, iks_sum: int, e0: int, delta: int, c):
    """Closed form for the arithmetic-progression generator e_i = e0 + i*delta mod r:
    sum_i k_i e_i = e0 * sum_i k_i + delta * sum_i i*k_i  (mod r).
    Callers pass the two integer sums (exact, however they were accumulated)."""
    t = (e0 * ks_sum + delta * iks_sum) % c.r
    return ec.mul(t, c.G, c)
