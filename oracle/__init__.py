"""CPU oracle for the cuMF_SGD hot path.  TEST INFRASTRUCTURE ONLY (see oracle/oracle.h)."""
