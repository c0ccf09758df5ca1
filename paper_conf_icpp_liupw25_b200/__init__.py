"""B200-native GBDT-MO hot path (Liu, Peng, Wen, ICPP'25): histogram building, sibling
subtraction and multi-output split search behind the C ABI of include/gbdtmo.h."""
from ._abi import Context, Problem, GbdtmoError, LOSS_MSE, LOSS_SOFTMAX, lib  # noqa: F401
from .booster import (Params, Dataset, Booster, PeerExchangeError, bin_features, bin_features_host,  # noqa: F401
                      bin_features_csc, train, predict)
from . import parallel  # noqa: F401
