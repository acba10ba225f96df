"""ORACLE -- test infrastructure only.

A plain, slow fp64 CPU forward pass of the Tonic networks, written from the paper
(sec 3) and the Caffe layer definitions it relies on (L77-78).
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import it.  It never imports the product package and
the product package never imports it.

Parity pins for every function live in ``tests/test_oracle_*.py`` (``-m "not gpu"``).
"""
from .ops import lib, build  # noqa: F401
from .net import OracleNet, parse_prototxt  # noqa: F401
