"""Probe: run one MNT4-753 debug_ec batch (argv: indices op) — for compute-sanitizer."""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
from tests.test_gpu_layers import _z_words  # noqa: E402
from tests.helpers import progression, points_to_words, words_to_point  # noqa: E402
from oracle import ec  # noqa: E402
from oracle.curves import CURVES  # noqa: E402
from paper_conf_asplos_ji0x024_b200 import msm  # noqa: E402
name = "mnt4_753"
idx = [int(v) for v in sys.argv[1].split(",")]
op = int(sys.argv[2])
c = CURVES[name]
Ps = list(progression(name, 24, 11)[0])
P = Ps[:12] + [Ps[0], Ps[1], None, Ps[2], None]
Q = Ps[12:24] + [Ps[0], ec.neg(Ps[1], c), Ps[3], None, None]
P = [P[i] for i in idx]
Q = [Q[i] for i in idx]
z = _z_words(c, 17, 5)[idx]
got = msm.debug_ec(name, op, points_to_words(P, name), points_to_words(Q, name), z)
print(all(words_to_point(got[i], name) == (ec.add(P[i], Q[i], c) if op < 2 else ec.double(P[i], c)) for i in range(len(idx))))
