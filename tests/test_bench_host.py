"""Host logic of bench.py that runs without a GPU: the clock/throttle summary that decides
whether a bench line is kept (B200_PROFILING.md clocks rule)."""
import bench


def _row(sm, mx, hw=False, hw_th=False, sw_th=False, pcap=False):
    act = lambda b: "Active" if b else "Not Active"
    return ["0", str(sm), str(mx), "", "0x0", act(hw), act(hw_th), act(sw_th), act(pcap)]


def test_clock_summary_median_max_and_reasons():
    c = bench.ClockSampler(0)
    c.rows = [_row(1965, 1965), _row(1800, 1965, pcap=True), _row(1950, 1965), _row(1500, 1965, hw_th=True)]
    c.source = "nvml"
    s = c.summary()
    assert s["sm_mhz"] == (1800 + 1950) / 2
    assert s["sm_max_mhz"] == 1965
    assert s["reasons"] == ["hw_thermal_slowdown", "sw_power_cap"]
    assert s["samples"] == 4 and s["source"] == "nvml"


def test_clock_summary_nvidia_smi_rows_and_empty():
    c = bench.ClockSampler(0)
    # nvidia-smi csv row: index, sm, max, power, active mask, then the four reason columns
    c.rows = [["0", "1965", "1965", "650.1", "0x0000000000000000", "Not Active", "Not Active",
               "Active", "Not Active"]]
    assert c.summary()["reasons"] == ["sw_thermal_slowdown"]
    empty = bench.ClockSampler(0).summary()
    assert empty["samples"] == 0 and empty["sm_mhz"] is None and "source" in empty


def test_clock_sampler_maps_the_device_by_uuid():
    class FakeNvml:
        def __init__(self):
            self.calls = []

        def nvmlDeviceGetHandleByUUID(self, u):
            self.calls.append(("uuid", u))
            return "h-uuid"

        def nvmlDeviceGetHandleByIndex(self, i):
            self.calls.append(("index", i))
            return "h-index"

    nv = FakeNvml()
    c = bench.ClockSampler(3, uuid="GPU-1234", pci_bus_id="0000:1b:00.0")
    assert c._nvml_handle(nv) == "h-uuid" and nv.calls == [("uuid", "GPU-1234")]


def test_star_count_closed_form():
    # K_{1,s} embeddings = sum_v deg(v)^(falling s): K_6 (deg 5), ring C_7 (deg 2), star K_{1,4}
    from workloads import gen
    assert bench.star_count(gen.complete_graph(6), 3) == 6 * 5 * 4 * 3
    assert bench.star_count(gen.ring_graph(7), 2) == 7 * 2 * 1
    assert bench.star_count(gen.ring_graph(7), 3) == 0
    g = gen.query_from_edges(5, [(0, i) for i in range(1, 5)])
    star = gen.make_graph(5, [0, 0, 0, 0], [1, 2, 3, 4], None, 1)
    assert bench.star_count(star, 4) == 4 * 3 * 2 * 1 and g.nq == 5
