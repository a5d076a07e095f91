timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} 2>&1 | grep -E "Error|assert|FAILED|passed|failed|^E " | head -30
