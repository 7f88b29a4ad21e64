"""The tolerance helpers themselves: a corrupted element must fail (no NaN holes)."""
import numpy as np
import pytest

from oracle import Oracle
from tests.helpers import assert_update_close


@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_untouched_parameter_must_stay_put(opt):
    p_old = np.array([1.0, 0.5, -0.25], np.float32)
    g = np.array([0.0, 0.3, 0.0])          # elements 0 and 2 untouched (g_abs = 0)
    ga = np.abs(g)
    ref_p, ref_s = Oracle.update(opt, 0.1, p_old, g, None)
    kw = dict(got_s=ref_s, ref_s=ref_s, s_old=np.zeros(3)) if opt == "adagrad" else {}
    assert_update_close(ref_p, ref_p, p_old, g, ga, 0.1, opt, **kw)      # exact: passes
    bad = ref_p.copy()
    bad[0] = 1.7                                                          # untouched, corrupted
    with pytest.raises(AssertionError):
        assert_update_close(bad, ref_p, p_old, g, ga, 0.1, opt, **kw)
    bad = ref_p.copy()
    bad[1] += 0.05                                                        # touched, far off
    with pytest.raises(AssertionError):
        assert_update_close(bad, ref_p, p_old, g, ga, 0.1, opt, **kw)


def test_untouched_adagrad_state_must_stay_put():
    p_old = np.array([1.0, 0.5], np.float32)
    g = np.array([0.0, 0.3])
    ref_p, ref_s = Oracle.update("adagrad", 0.1, p_old, g, None)
    bad_s = ref_s.copy()
    bad_s[0] = 0.2
    with pytest.raises(AssertionError):
        assert_update_close(ref_p, ref_p, p_old, g, np.abs(g), 0.1, "adagrad", got_s=bad_s, ref_s=ref_s,
                            s_old=np.zeros(2))
