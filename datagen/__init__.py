"""Seeded synthetic-input generators shared by tests, bench and smoke (no method arithmetic)."""
from .rng import app_seed, round_to_grid  # noqa: F401
from .recipes import (INPUT_SHAPE, ROWS_PER_QUERY, gen_input_rows, gen_weights,  # noqa: F401
                      flat_blob, load_calib)
