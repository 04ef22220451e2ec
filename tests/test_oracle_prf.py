"""Pins for the counter-based input generator (X8) in the oracle.

sm64 is SplitMix64; its first outputs from states 0 and 1 are the published
reference values of the generator (Steele, Lea & Flood 2014 / Vigna's
splitmix64.c), so they pin the oracle's constants and shift amounts."""


def test_splitmix64_reference_outputs(oracle):
    assert oracle.sm64(0) == 0xE220A8397B1DCDAF
    assert oracle.sm64(1) == 0x910A2DEC89025CC1


def test_rand32_vectors(oracle):
    # X8 test vectors, computed there by an independent script
    assert [oracle.rand32(0, 0, i) for i in range(4)] == [0x4D197E6F, 0xC892B50E, 0xFF5FFA39, 0x20D09481]
    assert oracle.rand32(1, 1, 0) == 0xDE3C8082


def test_rand32_definition_by_composition(oracle):
    # RAND32(seed, tag, idx) = low32(sm(sm(seed) ^ (tag << 48) ^ idx)): composition of the pinned sm64
    for seed, tag, idx in [(5, 0, 7), (123456789, 3, 1 << 20), (2 ** 40 + 1, 0x8000, (17 << 20) + 5)]:
        want = oracle.sm64(oracle.sm64(seed) ^ (tag << 48) ^ idx) & 0xFFFFFFFF
        assert oracle.rand32(seed, tag, idx) == want
