"""ORACLE — test infrastructure only.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_hpdc_raschg18_b200`` never imports it, and it
shares no code with the product: the C++ oracle parses the spec JSON itself.

``run`` wraps the ``atf_oracle`` binary (built from atf_oracle.cpp with plain
g++); ``closed_forms`` holds the mathematical pins.
"""
