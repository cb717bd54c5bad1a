"""TEST INFRASTRUCTURE ONLY: the CPU oracle (see oracle/pem.hpp)."""
