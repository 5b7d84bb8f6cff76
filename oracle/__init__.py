"""CPU ORACLE — test infrastructure only.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import anything here. Nothing under oracle/ shares code with the product path
(paper_conf_eurosys_stratimk24_b200/); the product path never imports it.
"""
