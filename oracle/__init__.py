"""Oracle package — TEST INFRASTRUCTURE ONLY (see cagmres_oracle.py header)."""
