"""CPU oracle for the cusFFT sparse-FFT hot path.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
package.  The product path (``paper_conf_ipps_wangcc16_b200``) never imports it
and shares no code with it: no kernels, headers, helpers, tables or constant
generators.  See ``oracle/sfft_oracle.py`` for the citations.
"""
from .sfft_oracle import *  # noqa: F401,F403
