"""CPU oracle for the cuBLASTP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  The
product path (``paper_conf_ipps_zhangwlf14_b200``) never imports it, and this
package imports nothing from the product.

* ``oracle.oracle``   -- ctypes binding of the plain-C oracle (oracle.c).
* ``oracle.oracle_b`` -- a second, independent pure-Python formulation used to
  pin the C oracle on tiny inputs.
"""
