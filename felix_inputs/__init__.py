"""Seeded synthetic inputs shared by the oracle and the CUDA path (input generation only)."""
from .dag import *  # noqa: F401,F403
from .configs import (Config, MLPWeights, config, make_mlp, make_y0, var_upper_bounds,  # noqa: F401
                      c1_space, c2_space, c2_space_two_statements, c2_sketches, c5_space, bert_spaces, resnet50_spaces, paper_example_space,
                      mobilenet_v2_spaces,
                      DEFAULT_MLP, C1_MLP)
from .testspaces import allops_space, composite_space, rnan_space  # noqa: F401
