"""Host check of the fast-divmod magic numbers the kernels use for tile and
row decoding (decode/compute_base): compiled with g++ and
compared with exact division over all divisors < 70000 and 10^5 random ones."""
import os
import subprocess
import tempfile

HERE = os.path.dirname(os.path.abspath(__file__))


def test_fastdiv_matches_division():
    with tempfile.TemporaryDirectory() as d:
        exe = os.path.join(d, "fastdiv_check")
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-o", exe,
                               os.path.join(HERE, "cpp", "fastdiv_check.cpp")])
        out = subprocess.run([exe], capture_output=True, text=True)
        n, bad = map(int, out.stdout.split())
        assert out.returncode == 0 and bad == 0 and n > 1_000_000
