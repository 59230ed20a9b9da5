"""The AES-128 core netlist (workloads/aes.py; the paper's Table I circuit family)
simulated by the ORACLE: FIPS-197 Appendix C.1 known-answer vector (tests/golden) and an
independent textbook AES (tests/_aes_ref.py) on random keys / plaintexts (CPU only)."""
import os

import numpy as np

import oracle
from workloads import aes
from tests import _aes_ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fips197_c1.txt")


def _golden():
    d = {}
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        k, v = line.split(None, 1)
        d[k] = v.strip()
    return d


def test_sbox_table_matches_fips197():
    g = _golden()
    sb = aes.sbox_table()
    for pair in g["SBOX"].split():
        x, y = pair.split(":")
        assert sb[int(x, 16)] == int(y, 16)
    assert sb == _aes_ref.SBOX                       # two independent constructions


def test_reference_aes_known_answer():
    g = _golden()
    assert _aes_ref.encrypt(bytes.fromhex(g["KEY"]), bytes.fromhex(g["PLAINTEXT"])).hex() == g["CIPHERTEXT"]


def test_aes_netlist_on_oracle_known_answer_and_random():
    g = _golden()
    nl = aes.aes128_core()
    lanes = 128
    rng = np.random.default_rng(7)
    keys = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    pts = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    keys[0] = np.frombuffer(bytes.fromhex(g["KEY"]), dtype=np.uint8)
    pts[0] = np.frombuffer(bytes.fromhex(g["PLAINTEXT"]), dtype=np.uint8)
    stim = aes.aes_stimulus(keys, pts)
    o = oracle.simulate(nl, np.arange(lanes), 12, host_stim=stim, want=("last",))
    ct = aes.ciphertexts(o["last"])
    assert bytes(ct[0]).hex() == g["CIPHERTEXT"]
    for s in range(lanes):
        assert bytes(ct[s]) == _aes_ref.encrypt(bytes(keys[s]), bytes(pts[s])), s
    # the polynomial-network evaluation of the same 8-input LUTs agrees
    p = oracle.simulate(nl, np.arange(64), 12, host_stim=stim, mode="poly", want=("last",))
    assert p["violations"] == 0 and np.array_equal(p["last"], o["last"][:64])
