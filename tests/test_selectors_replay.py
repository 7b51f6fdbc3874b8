"""Pins for the selector replays in oracle/selectors.py.

Expected modes are worked by hand from the prose of Alg. 4
and Alg. 5; readings R5-R7.
"""
import math

from oracle import selectors as sel

WE, EP = sel.WE, sel.EP


def test_constants_from_paper():
    assert (sel.ALPHA, sel.BETA) == (768, 512)
    assert (sel.N_SAMPS, sel.GAMMA) == (512, 4.0)
    assert sel.EP_MIN_FRONTIER == 512


def test_hybrid_worked_example():
    # L0 starts WE; |5-1| <= 768 keep; |900-5| > 768 and 900 > 512 -> EP;
    # |2000-900| > 768, 2000 > 512 -> EP; |300-2000| > 768, 300 <= 512 -> WE;
    # |2-300| <= 768 keep WE.
    assert sel.hybrid_modes([1, 5, 900, 2000, 300, 2]) == [WE, WE, EP, EP, WE, WE]


def test_hybrid_change_exactly_alpha_keeps_mode():
    # Q_change == alpha is "less than or equal" -> keep
    assert sel.hybrid_modes([1, 769, 1]) == [WE, WE, WE]
    assert sel.hybrid_modes([1, 770, 1]) == [WE, EP, WE]


def test_hybrid_beta_is_strict():
    # Q_next_len must be LARGER than beta
    assert sel.hybrid_modes([1000, 512 - 0, 2000])[1] == WE   # change 488: keep WE anyway
    assert sel.hybrid_modes([2000, 512, 5]) == [WE, WE, WE]    # change 1488, 512 !> 512 -> WE


def test_hybrid_high_diameter_stays_we():
    assert sel.hybrid_modes([1, 4, 8, 12] + [16] * 300) == [WE] * 304


def test_sampling_median_and_threshold():
    n = 1 << 18                       # gamma*log2(n) = 72
    assert math.isclose(sel.GAMMA * math.log2(n), 72.0)
    assert sel.sampling_decision([6] * 300 + [400] * 212, n) is True     # median 6
    assert sel.sampling_decision([6] * 200 + [400] * 312, n) is False    # median 400
    assert sel.sampling_decision([71] * 3, n) is True and sel.sampling_decision([72] * 3, n) is False
    assert sel.sampling_decision([], n) is False                          # WE by default
    # median = keys[n'/2] after an ascending sort: 4 samples -> index 2
    assert sel.sampling_decision([100, 1, 2, 100], n) is False
    assert sel.sampling_decision([1, 2, 3, 100], n) is True


def test_sampling_guard():
    assert sel.sampling_modes([1, 700, 511, 512, 3], True) == [WE, EP, WE, EP, WE]
    assert sel.sampling_modes([1, 700, 3], False) == [WE, WE, WE]
