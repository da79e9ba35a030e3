"""ORACLE -- test infrastructure only.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` leg may import anything under ``oracle/``.  The product
package ``paper_conf_icpp_yecrbypnmskn24_b200`` never imports it and shares no
code with it.

* ``oracle.transfer`` -- ctypes wrapper of ``viper_oracle.c`` (plain C: LAY,
  CKS, pack, seal, deliver, verify, double buffer, atomic swap, acquire/release).
* ``oracle.sched_ref`` -- numpy/scipy rendition of the paper's Inference
  Performance Predictor: TLP fits (s4.3 P:1284-1328), Eq. 1-3,
  Algorithms 1-3.
"""
